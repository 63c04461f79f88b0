#!/usr/bin/env python
"""List SASS instructions with excess shared-memory wavefronts (bank conflicts)
from `ncu -i X --page source --csv --print-source=cuda,sass`."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
long_hdr = max((r for r in rows if r and r[0] == "Line No"), key=len)
iE = long_hdr.index("L1 Wavefronts Shared Excessive")
iW = long_hdr.index("L1 Wavefronts Shared")
iI = long_hdr.index("L1 Wavefronts Shared Ideal")
func = fpath = line = src = None
res = []
tot = {}
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fpath = r[1].split("/")[-1]; continue
    if r[0] == "Function Name":
        func = r[1].replace("void bcf::", "").split(">(")[0] + ">"; continue
    if r[0] == "Line No":
        continue
    if r[0]:
        line, src = r[0], r[1]
    if len(r) != len(long_hdr) or not r[2].startswith("0x"):
        continue
    try:
        ex = int(r[iE] or 0); wf = int(r[iW] or 0); ideal = int(r[iI] or 0)
    except ValueError:
        continue
    t = tot.setdefault(func, [0, 0, 0]); t[0] += ex; t[1] += wf; t[2] += ideal
    if ex > 0:
        res.append((ex, wf, func, f"{fpath}:{line}", src.strip()[:60], r[3].strip()[:50]))
for f, (ex, wf, ideal) in tot.items():
    print(f"{f}: smem wavefronts {wf} ideal {ideal} excessive {ex}")
for x in sorted(res, reverse=True)[: int(sys.argv[2]) if len(sys.argv) > 2 else 30]:
    print(x)
