"""Per-configuration sums of the unit-level shared-memory counters from an ncu
raw CSV (`ncu -i X --page raw --csv --metrics ...`) and the launch map written
by tools/conflicts.py."""
import csv
import json
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[0]
data = [r for r in rows[2:] if len(r) == len(hdr)]
mp = json.load(open(sys.argv[2]))
col = {h: i for i, h in enumerate(hdr)}


def num(r, m):
    v = r[col[m]].replace(",", "")
    try:
        return float(v)
    except ValueError:
        return 0.0


metrics = [m for m in hdr if m.startswith("l1tex__") or m.startswith("gpu__time")]
print("config kind kernel launches " + " ".join(m.replace("l1tex__data_bank_conflicts_pipe_lsu_mem_shared", "conf")
                                              .replace("l1tex__data_pipe_lsu_wavefronts_mem_shared", "wf")
                                              for m in metrics))
for e in mp:
    sel = data[e["first_launch"]:e["first_launch"] + e["launches"]]
    by = {}
    for r in sel:
        k = r[col["Kernel Name"]].split("<")[0].split("::")[-1] if "Kernel Name" in col else "k"
        acc = by.setdefault(k, [0] + [0.0] * len(metrics))
        acc[0] += 1
        for i, m in enumerate(metrics):
            acc[i + 1] += num(r, m)
    for k, acc in by.items():
        print(f"{e['algo']}:{e['E']}:{e['u']} {e['kind']} {k} {acc[0]} " + " ".join(f"{v:.0f}" for v in acc[1:]))
