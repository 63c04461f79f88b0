#!/bin/bash
# round-1 probe: TMA/mbarrier counter calibration, full capture of the
# default merge pass + block sort (traffic, source-level smem excess), and
# E = 31 bench lines at u = 128 / 256 / 512 (kernel split per variant)
set -u
mkdir -p gpurun_out /tmp/ev
M="l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,smsp__inst_executed_op_ldsm.sum"
timeout 300 ncu --metrics $M --csv --log-file gpurun_out/calib_tma.csv ./tools/ncu_calib_tma > gpurun_out/calib_tma.log 2>&1
if [[ " $* " == *" full "* ]]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"block_sort|merge_pass" -s 14 -c 3 -o /tmp/ev/full -f python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/ev_full.log 2>&1
ncu -i /tmp/ev/full.ncu-rep --page raw --csv > gpurun_out/ev_full_raw.csv 2>&1
ncu -i /tmp/ev/full.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/ev/full_src.csv 2>&1
python tools/smem_excess.py /tmp/ev/full_src.csv 20 > gpurun_out/ev_excess.txt 2>&1
python tools/src_hot.py /tmp/ev/full_src.csv 40 0 > gpurun_out/ev_hot_k0.txt 2>&1
python tools/src_hot.py /tmp/ev/full_src.csv 40 1 > gpurun_out/ev_hot_k1.txt 2>&1
fi
for u in ${PROBE_U:-128 256 512}; do
  timeout 300 python bench.py --E 31 --u $u --steps 60 --no-extras 2>gpurun_out/bench_u$u.err | tail -1 > gpurun_out/bench_E31_u$u.json
done
echo done
