#!/bin/bash
# GPU parity (fail fast) + full bench + counter calibration
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x --timeout 300 --tb=short > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
M="l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"
[ -x tools/ncu_calib_tma ] && [ -n "${CALIB:-}" ] && timeout 300 ncu --metrics $M --csv --log-file gpurun_out/calib_tma4.csv ./tools/ncu_calib_tma > gpurun_out/calib_tma4.log 2>&1
echo done
