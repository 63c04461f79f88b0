#!/bin/bash
# One GPU session on the gpurun box; every output lands in gpurun_out/
# (merged back by gpurun).  Modes run in the order given:
#   tests      pytest -m gpu
#   bench      python bench.py (default N=1 line) -> bench.json
#   launches   ncu launch list (gpu__time_duration, cold, serialised) of a short bench
#   conflicts  ncu unit-level smem conflict / wavefront / DRAM counters (tools/conflicts.py; CONF_ARGS)
#   full       ncu --set full of one merge pass and one block sort -> .ncu-rep
#   evidence   launch list + full capture + SASS-level smem excess (random and worst case)
#   ab         bench summary line per library variant (VARIANTS="a b" -> build_variants/lib_<v>.so; CFGS)
#   "<cmd>"    anything else is run by bash
set -u
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out /tmp/ev
M="l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ldgsts.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/gpu_info.txt 2>&1
for what in "$@"; do
  case "$what" in
    tests)
      timeout 2400 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" ;;
    bench)
      timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" ;;
    launches)
      timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
        python bench.py --steps 4 --warmup 3 --no-extras > gpurun_out/launches_bench.json 2>&1; echo "launches rc=$?" ;;
    conflicts)
      timeout 1200 ncu --metrics $M --clock-control none -k regex:"block_sort|merge_pass" --csv --log-file gpurun_out/conflicts.csv \
        python tools/conflicts.py ${CONF_ARGS:-} > gpurun_out/conflicts.log 2>&1; echo "conflicts rc=$?" ;;
    full)
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:merge_pass -s 6 -c 1 -o gpurun_out/prof_merge -f \
        python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/prof_merge.log 2>&1
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:block_sort -s 2 -c 1 -o gpurun_out/prof_block -f \
        python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/prof_block.log 2>&1; echo "full rc=$?" ;;
    evidence)
      timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
        python bench.py --steps 4 --warmup 3 --no-extras > /dev/null 2>&1
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:"block_sort|merge_pass" -s 14 -c 3 -o /tmp/ev/full -f \
        python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/ev_full.log 2>&1
      ncu -i /tmp/ev/full.ncu-rep --page raw --csv > gpurun_out/ev_full_raw.csv 2>&1
      ncu -i /tmp/ev/full.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/ev/full_src.csv 2>&1
      python tools/smem_excess.py /tmp/ev/full_src.csv 20 > gpurun_out/ev_excess.txt 2>&1
      python tools/src_hot.py /tmp/ev/full_src.csv 40 0 > gpurun_out/ev_hot_k0.txt 2>&1
      python tools/src_hot.py /tmp/ev/full_src.csv 40 1 > gpurun_out/ev_hot_k1.txt 2>&1
      timeout 900 ncu --section SourceCounters --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,gpu__time_duration.sum \
        -k regex:"block_sort|merge_pass" -o /tmp/ev/conf -f python tools/conflicts.py --n 16777216 --kinds random,worst \
        --configs ${EV_CONFIGS:-cf:31:128,base:31:128,cf:15:256,base:15:256} --out gpurun_out/ev_conf_map.json > gpurun_out/ev_conf.log 2>&1
      ncu -i /tmp/ev/conf.ncu-rep --page raw --csv --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,gpu__time_duration.sum \
        > gpurun_out/ev_conf_raw.csv 2>&1
      ncu -i /tmp/ev/conf.ncu-rep --page source --csv --print-source=cuda,sass > /tmp/ev/conf_src.csv 2>&1
      python tools/smem_excess.py /tmp/ev/conf_src.csv 40 > gpurun_out/ev_conf_excess.txt 2>&1; echo "evidence done" ;;
    ab)
      for v in ${VARIANTS:-}; do
        for cfg in ${CFGS:-31_128}; do
          set -- ${cfg//_/ }
          BCF_LIB=build_variants/lib_$v.so timeout 300 python bench.py --E $1 --u $2 --steps ${AB_STEPS:-100} --no-extras 2>&1 | tail -1 | \
            python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('$v','E',d['config']['E'],'u',d['config']['u'],'Gk/s %.2f'%(d['value']/1e9),'w/r %.4f'%d['worst_over_random_time'],'block %.1fus'%(1e3*k['block_sort']['avg_ms']),'merge %.1fus'%(1e3*k['merge_pass']['avg_ms']),'frac %.3f'%d['roofline']['frac'])" \
            >> gpurun_out/ab.txt 2>&1 || echo "$v failed" >> gpurun_out/ab.txt
        done
      done; echo "ab done" ;;
    *) bash -c "$what"; echo "custom rc=$?" ;;
  esac
done
