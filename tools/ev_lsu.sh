set -u
mkdir -p gpurun_out /tmp/ev
MET=l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,gpu__time_duration.sum
for mode in notma tma; do
  if [ $mode = notma ]; then export BCF_NO_TMA=1; else unset BCF_NO_TMA; fi
  timeout 900 ncu --section SourceCounters --metrics $MET -k regex:"block_sort|merge_pass" -o /tmp/ev/conf_$mode -f \
    python tools/conflicts.py --n 4194304 --kinds random,worst --configs cf:31:128,cf:16:128,cf:8:256,cf:12:128,cf:15:256 \
    --out gpurun_out/ev_map_$mode.json > gpurun_out/ev_$mode.log 2>&1
  ncu -i /tmp/ev/conf_$mode.ncu-rep --page raw --csv --metrics $MET > gpurun_out/ev_raw_$mode.csv 2>&1
  ncu -i /tmp/ev/conf_$mode.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/ev/src_$mode.csv 2>&1
  python tools/smem_excess.py /tmp/ev/src_$mode.csv 40 > gpurun_out/ev_excess_$mode.txt 2>&1
done
echo done
