"""Per-configuration sums of the unit-level shared-memory counters from an ncu
`--metrics ... --csv --log-file` capture (one row per launch and metric) and
the launch map written by tools/conflicts.py."""
import csv
import json
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 14 and r[0].isdigit()]
mp = json.load(open(sys.argv[2]))
launch = defaultdict(dict)
names = {}
for r in rows:
    launch[int(r[0])][r[12]] = float(r[14].replace(",", "") or 0)
    names[int(r[0])] = r[4].split("<")[0].replace("void ", "").split("::")[-1]
ids = sorted(launch)
short = lambda m: (m.replace("l1tex__data_bank_conflicts_pipe_lsu_mem_shared", "conf")  # noqa: E731
                   .replace("l1tex__data_pipe_lsu_wavefronts_mem_shared", "wf").replace(".sum", ""))
metrics = sorted({m for d in launch.values() for m in d})
print("%-14s %-6s %-22s %3s " % ("config", "kind", "kernel", "n") + " ".join("%12s" % short(m) for m in metrics))
for e in mp:
    sel = ids[e["first_launch"]:e["first_launch"] + e["launches"]]
    by = defaultdict(lambda: [0, defaultdict(float)])
    for i in sel:
        b = by[names[i]]
        b[0] += 1
        for m, v in launch[i].items():
            b[1][m] += v
    for k, (cnt, acc) in by.items():
        cfg = f"{e['algo']}:{e['E']}:{e['u']}"
        print("%-14s %-6s %-22s %3d " % (cfg, e["kind"], k, cnt) + " ".join("%12.0f" % acc[m] for m in metrics))
