#!/usr/bin/env python
"""Summarise an `ncu --page raw --csv` export of a --set full capture into the
per-kernel JSON kept under profiles/ (time, DRAM bytes, issue activity,
occupancy limits, instructions, bank conflicts, L2 hit rate, stall reasons
per issued instruction)."""
import csv, json, sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, units = rows[0], rows[1]
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "lts__t_sector_hit_rate.pct",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed"]
out = []
for r in rows[2:]:
    d = {"kernel": r[hdr.index("Kernel Name")]}
    for k in keys:
        for i, h in enumerate(hdr):
            if h.endswith(k) and r[i]:
                d[k] = (r[i] + " " + units[i]).strip()
                break
    st = {}
    for i, h in enumerate(hdr):
        if "smsp__average_warps_issue_stalled_" in h and h.endswith("_per_issue_active.ratio") and r[i]:
            name = h.split("smsp__average_warps_issue_stalled_")[1].replace("_per_issue_active.ratio", "")
            v = float(r[i])
            if v >= 0.2:
                st[name] = round(v, 2)
    d["stalls_per_issue"] = st
    out.append(d)
json.dump(out, sys.stdout, indent=1)
