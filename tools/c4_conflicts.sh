# BASELINE config C4 conflict evidence over every instantiated (E, u):
#  (1) unit counter, one CTA per SM, LSU-only (BCF_ONE_CTA_PER_SM=1), CF, 2^27 worst case + random
#  (2) unit counter, default kernels, CF and baseline, 2^27
#  (3) SASS-level excessive wavefronts (SourceCounters), CF and baseline, 2^22
set -u
mkdir -p gpurun_out /tmp/c4
MET=l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,gpu__time_duration.sum
CF=""; BASE=""
for E in 7 8 9 10 11 12 13 14 15 16 17 31; do for u in 128 256 512; do CF="$CF,cf:$E:$u"; BASE="$BASE,base:$E:$u"; done; done
CF=${CF#,}; BASE=${BASE#,}
BCF_ONE_CTA_PER_SM=1 BCF_NO_PDL=1 timeout 3000 ncu --metrics $MET -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/c4_onecta.csv \
  python tools/conflicts.py --n 134217728 --kinds random,worst --configs $CF --out gpurun_out/c4_map_onecta.json > gpurun_out/c4_onecta.log 2>&1
echo "onecta rc=$?"
timeout 3000 ncu --metrics $MET -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/c4_default.csv \
  python tools/conflicts.py --n 134217728 --kinds random,worst --configs $CF,$BASE --out gpurun_out/c4_map_default.json > gpurun_out/c4_default.log 2>&1
echo "default rc=$?"
timeout 3000 ncu --section SourceCounters --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum -k regex:"block_sort|merge_pass" -o /tmp/c4/sass -f \
  python tools/conflicts.py --n 4194304 --kinds random,worst --configs $CF,$BASE --out gpurun_out/c4_map_sass.json > gpurun_out/c4_sass.log 2>&1
echo "sass rc=$?"
ncu -i /tmp/c4/sass.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/c4/sass_src.csv 2>&1
python tools/smem_excess.py /tmp/c4/sass_src.csv 60 > gpurun_out/c4_sass_excess.txt 2>&1
python tools/conf_table2.py gpurun_out/c4_onecta.csv gpurun_out/c4_map_onecta.json > gpurun_out/c4_table_onecta.txt 2>&1
python tools/conf_table2.py gpurun_out/c4_default.csv gpurun_out/c4_map_default.json > gpurun_out/c4_table_default.txt 2>&1
echo done
