#!/usr/bin/env python
"""Per-CUDA-source-line totals from
`ncu -i X.ncu-rep --page source --csv --print-source=cuda,sass` (first kernel)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
which = int(sys.argv[3]) if len(sys.argv) > 3 else 0
out, fpath, hdr, kern = [], None, None, -1
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fpath = r[1].split("/")[-1]
        continue
    if r[0] == "Function Name":
        if r[1] != globals().get("_cur"):
            globals()["_cur"] = r[1]
            kern += 1
        continue
    if kern != which:
        continue
    if r[0] == "Line No":
        hdr = r
        iX = hdr.index("Instructions Executed")
        iS = hdr.index("Warp Stall Sampling (All Samples)")
        continue
    if hdr and r[0].isdigit():
        try:
            x = int(r[iX] or 0)
            s = int(r[iS] or 0)
        except ValueError:
            continue
        out.append((x, s, fpath, int(r[0]), r[1].strip()[:80]))
tot = sum(o[0] for o in out) or 1
tots = sum(o[1] for o in out) or 1
print("total warp instructions", tot, "stall samples", tots)
for o in sorted(out, key=lambda o: -o[0])[:n]:
    print(f"{o[0]:>10} {100*o[0]/tot:5.1f}% stall={100*o[1]/tots:5.1f}% {o[2]}:{o[3]} {o[4]}")
