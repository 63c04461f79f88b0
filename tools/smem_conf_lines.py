#!/usr/bin/env python
"""SASS instructions with shared-memory bank conflicts (any per-instruction
conflict / excess column) from `ncu -i X --page source --csv
--print-source=cuda,sass`: prints the header columns it used and the top
instructions per kernel."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
long_hdr = max((r for r in rows if r and r[0] == "Line No"), key=len)
cols = [i for i, h in enumerate(long_hdr) if ("Shared" in h and ("Conflict" in h or "Excess" in h))]
print("columns:", [long_hdr[i] for i in cols])
func = fpath = line = src = None
res = []
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fpath = r[1].split("/")[-1]
        continue
    if r[0] == "Function Name":
        func = r[1].replace("void bcf::", "").split(">(")[0] + ">"
        continue
    if r[0] == "Line No":
        continue
    if r[0]:
        line, src = r[0], r[1]
    if len(r) != len(long_hdr) or not r[2].startswith("0x"):
        continue
    vals = []
    for i in cols:
        try:
            vals.append(int(float(r[i] or 0)))
        except ValueError:
            vals.append(0)
    nway = vals[0] if len(vals) > 0 else 0
    excess = sum(vals[1:])
    if nway > 1 or excess > 0:
        res.append((max(vals), vals, func, f"{fpath}:{line}", (src or "").strip()[:70], r[3].strip()[:60]))
for x in sorted(res, reverse=True)[:top]:
    print(x)
print("instructions with nonzero:", len(res))
