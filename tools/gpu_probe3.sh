#!/bin/bash
# bench with the configs[2] legs; unit-level conflicts of the default (31,128)
# with the TMA merge pass and with BCF_NO_TMA=1 (LSU-only per-tile merge pass)
mkdir -p gpurun_out
M="l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 600 ncu --metrics $M --clock-control none -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/conf_tma.csv python tools/conflicts.py --configs cf:31:128,base:31:128 --out gpurun_out/conf_tma_map.json > gpurun_out/conf_tma.log 2>&1
BCF_NO_TMA=1 timeout 600 ncu --metrics $M --clock-control none -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/conf_notma.csv python tools/conflicts.py --configs cf:31:128 --out gpurun_out/conf_notma_map.json > gpurun_out/conf_notma.log 2>&1
BCF_NO_TMA=1 timeout 300 python bench.py --steps 60 --no-extras 2>/dev/null | tail -1 > gpurun_out/bench_notma.json
echo done
