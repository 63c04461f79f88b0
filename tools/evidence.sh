#!/bin/bash
# ncu evidence for the default configuration (outputs small summaries only)
set -u
mkdir -p gpurun_out /tmp/ev
# 1. launch list of a short bench run (cold, serialised)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 4 --warmup 3 --no-extras > /dev/null 2>&1
# 2. full capture: block sort + one merge pass (random input, step 0 of the timed run)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"block_sort|merge_pass" -s 14 -c 3 -o /tmp/ev/full -f python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/ev_full.log 2>&1
ncu -i /tmp/ev/full.ncu-rep --page raw --csv > gpurun_out/ev_full_raw.csv 2>&1
ncu -i /tmp/ev/full.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/ev/full_src.csv 2>&1
python tools/smem_excess.py /tmp/ev/full_src.csv 20 > gpurun_out/ev_excess.txt 2>&1
python tools/src_hot.py /tmp/ev/full_src.csv 40 0 > gpurun_out/ev_hot_k0.txt 2>&1
python tools/src_hot.py /tmp/ev/full_src.csv 40 1 > gpurun_out/ev_hot_k1.txt 2>&1
# 3. worst-case input: SASS-level smem excess for the whole sort (source counters)
timeout 900 ncu --section SourceCounters --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,gpu__time_duration.sum -k regex:"block_sort|merge_pass" -o /tmp/ev/conf -f python tools/conflicts.py --n 16777216 --kinds random,worst --configs ${EV_CONFIGS:-cf:31:128,base:31:128,cf:15:256,base:15:256} --out gpurun_out/ev_conf_map.json > gpurun_out/ev_conf.log 2>&1
ncu -i /tmp/ev/conf.ncu-rep --page raw --csv --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,gpu__time_duration.sum > gpurun_out/ev_conf_raw.csv 2>&1
ncu -i /tmp/ev/conf.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/ev/conf_src.csv 2>&1
python tools/smem_excess.py /tmp/ev/conf_src.csv 40 > gpurun_out/ev_conf_excess.txt 2>&1
echo done
