# unit-level smem conflict counter: default kernels vs the one-CTA-per-SM LSU-only mode
set -u
mkdir -p gpurun_out /tmp/ev
MET=l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ldgsts.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,gpu__time_duration.sum
CFG=${CFG:-cf:31:128,cf:16:128,cf:8:256,cf:12:128,cf:15:256,cf:17:256,base:31:128,base:15:256}
N=${N:-4194304}
BCF_ONE_CTA_PER_SM=1 BCF_NO_PDL=1 timeout 1200 ncu --metrics $MET -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/zero_onecta.csv \
  python tools/conflicts.py --n $N --kinds random,worst --configs $CFG --out gpurun_out/zero_map_onecta.json > gpurun_out/zero_onecta.log 2>&1
timeout 1200 ncu --metrics $MET -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/zero_default.csv \
  python tools/conflicts.py --n $N --kinds random,worst --configs $CFG --out gpurun_out/zero_map_default.json > gpurun_out/zero_default.log 2>&1
echo done
