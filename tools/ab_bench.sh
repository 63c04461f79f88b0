#!/bin/bash
# A/B: bench line summary for each library variant given as NAME=PATH args
for spec in "$@"; do
  name=${spec%%=*}; lib=${spec#*=}
  for cfg in ${CFGS:-15_256}; do
    set -- ${cfg//_/ }
    BCF_LIB=$lib timeout 200 python bench.py --E $1 --u $2 --steps 100 --no-extras 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('$name','E',d['config']['E'],'u',d['config']['u'],'Gk/s %.2f'%(d['value']/1e9),'w/r %.4f'%d['worst_over_random_time'],'block %.1fus'%(1e3*k['block_sort']['avg_ms']),'merge %.1fus'%(1e3*k['merge_pass']['avg_ms']),'frac %.3f'%d['roofline']['frac'])" || echo "$name failed"
  done
done
