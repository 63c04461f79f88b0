#!/bin/bash
# One GPU session: tests, bench, ncu evidence.  Outputs under gpurun_out/.
set -u
mkdir -p gpurun_out
M="l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"
if [[ " $* " == *" tests "* ]]; then
  timeout 1500 python -m pytest tests -q -m gpu --timeout 600 --tb=short > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
fi
if [[ " $* " == *" bench "* ]]; then
  timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
fi
if [[ " $* " == *" launches "* ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 4 --warmup 3 --no-extras > gpurun_out/launches_bench.json 2>&1
fi
if [[ " $* " == *" conflicts "* ]]; then
  timeout 900 ncu --metrics $M --clock-control none -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/conflicts.csv python tools/conflicts.py ${CONF_ARGS:-} > gpurun_out/conflicts.log 2>&1
fi
if [[ " $* " == *" full "* ]]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:merge_pass -s 6 -c 1 -o gpurun_out/prof_merge -f python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/prof_merge.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:block_sort -s 2 -c 1 -o gpurun_out/prof_block -f python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/prof_block.log 2>&1
fi
echo done
