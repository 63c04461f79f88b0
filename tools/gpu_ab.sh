#!/bin/bash
# calibration (TMA/mbarrier/STS cases) + A/B of library variants in build_variants/
mkdir -p gpurun_out
M="l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"
[ -x tools/ncu_calib_tma ] && timeout 300 ncu --metrics $M --csv --log-file gpurun_out/calib_tma3.csv ./tools/ncu_calib_tma > gpurun_out/calib_tma3.log 2>&1
args=""
for v in ${VARIANTS}; do args="$args $v=build_variants/lib_$v.so"; done
CFGS=${CFGS:-31_128} bash tools/ab_bench.sh $args > gpurun_out/ab.txt 2>&1
CFGS=${CFGS:-31_128} bash tools/ab_bench.sh $args >> gpurun_out/ab.txt 2>&1
echo done
