# SASS-level (per-instruction) smem excess for every instantiated CF (E, u) and the
# baseline, one ncu SourceCounters capture per configuration (random + worst case)
set -u
mkdir -p gpurun_out
N=${N:-1048576}
for c in ${CFGS}; do
  timeout 600 ncu --section SourceCounters --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum -k regex:"merge_pass|block_sort" \
    -o /tmp/c4s -f python tools/conflicts.py --n $N --kinds random,worst --configs $c --out /tmp/c4s.json > /dev/null 2>&1
  ncu -i /tmp/c4s.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/c4s.csv 2>&1
  echo "## $c"
  python tools/smem_excess.py /tmp/c4s.csv 3 | cut -c1-220
done
