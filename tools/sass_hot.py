#!/usr/bin/env python
"""Summarise an ncu --page source --print-source=sass CSV: total executed warp
instructions, and the hottest address ranges (loops)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
iA, iS, iX = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed")
iT = hdr.index("Warp Stall Sampling (All Samples)")
data = []
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    try:
        data.append((int(r[iA], 16) if r[iA].startswith("0x") else int(r[iA]), r[iS], int(r[iX] or 0), int(r[iT] or 0)))
    except ValueError:
        pass
tot = sum(d[2] for d in data)
stall = sum(d[3] for d in data)
print("total warp instructions executed:", tot, " samples:", stall)
# segment by executed count level
seg = []
cur = None
for a, s, x, t in data:
    if cur and abs(x - cur[2]) <= 0.05 * max(x, cur[2], 1):
        cur[1] = a; cur[3] += x; cur[4] += 1; cur[5] += t
    else:
        if cur: seg.append(cur)
        cur = [a, a, x, x, 1, t, s]
seg.append(cur)
seg.sort(key=lambda c: -c[3])
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
for c in seg[:n]:
    print(f"{c[0]:#07x}-{c[1]:#07x} n={c[4]:4d} each~{c[2]:>10d} sum={c[3]:>12d} ({100*c[3]/tot:5.1f}%) samples={c[5]:6d} first: {c[6][:60]}")
