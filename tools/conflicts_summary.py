#!/usr/bin/env python
"""Summarise an ncu --csv metric log of tools/conflicts.py into per-configuration
bank-conflict totals (CF vs baseline, random vs worst-case)."""
import csv, json, sys
from collections import defaultdict
rows = list(csv.reader(open(sys.argv[1])))
mapping = json.load(open(sys.argv[2]))
hdr = None
data = []
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        data.append(d)
# group by launch ID
by_id = defaultdict(dict)
names = {}
for d in data:
    i = int(d["ID"])
    v = d["Metric Value"].replace(",", "")
    try:
        v = float(v)
    except ValueError:
        continue
    by_id[i][d["Metric Name"]] = v
    names[i] = d["Kernel Name"]
ids = sorted(by_id)
out = []
for m in mapping:
    sel = ids[m["first_launch"]:m["first_launch"] + m["launches"]]
    agg = defaultdict(float)
    for i in sel:
        for k, v in by_id[i].items():
            agg[k] += v
    bc = agg.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", float("nan"))
    wf_ld = agg.get("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", 0)
    wf_st = agg.get("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum", 0)
    n_ld = agg.get("smsp__sass_inst_executed_op_shared_ld.sum", 0)
    n_st = agg.get("smsp__sass_inst_executed_op_shared_st.sum", 0)
    dram = agg.get("dram__bytes_read.sum", 0) + agg.get("dram__bytes_write.sum", 0)
    t = agg.get("gpu__time_duration.sum", 0)
    rec = dict(m)
    rec.update({"bank_conflicts": bc,
                "conflicts_ld": agg.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum"),
                "conflicts_st": agg.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum"),
                "smem_ld_inst": n_ld, "smem_st_inst": n_st,
                "wavefronts_per_ld": wf_ld / n_ld if n_ld else None,
                "dram_bytes": dram, "kernel_time_ns_sum": t,
                "kernels": sorted(set(names[i].split("(")[0] for i in sel))})
    out.append(rec)
for r in out:
    print(f'{r["algo"]:4s} E={r["E"]:2d} u={r["u"]:3d} {r["kind"]:6s} conflicts={r["bank_conflicts"]:>12.0f} '
          f'(ld {r["conflicts_ld"]:.0f}, st {r["conflicts_st"]:.0f}) wf/ld={r["wavefronts_per_ld"]:.3f} '
          f'launches={r["launches"]} time_sum={r["kernel_time_ns_sum"]/1e3:.1f}us')
if len(sys.argv) > 3:
    json.dump(out, open(sys.argv[3], "w"), indent=1)
