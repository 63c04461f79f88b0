#!/bin/bash
set -e; python paper_conf_spaa_berneys25_b200/build.py > /dev/null; set +e
# quick: parity subset + bench lines for a few (E,u)
timeout 600 python -m pytest tests/test_gpu_sort.py -q -m gpu -x --timeout 300 -k "not full" 2>&1 | tail -2
for cfg in ${CFGS:-15_256 17_256 15_512 16_256}; do
  cfg=${cfg//_/ }
  set -- $cfg
  timeout 300 python bench.py --E $1 --u $2 --steps 100 --no-extras 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('E',d['config']['E'],'u',d['config']['u'],'Gk/s %.2f'%(d['value']/1e9),'w/r %.4f'%d['worst_over_random_time'],'block %.1fus'%(1e3*k['block_sort']['avg_ms']),'merge %.1fus'%(1e3*k['merge_pass']['avg_ms']),'frac %.3f'%d['roofline']['frac'], 'clk', d['clocks']['sm_mhz'])"
done
