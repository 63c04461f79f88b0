#!/bin/bash
# A/B of environment settings on the default bench line (one summary line each).
# usage: tools/ab_env.sh "LABEL1:VAR=x VAR2=y" "LABEL2:VAR=z" ...   (env AB_ARGS: extra bench args)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for spec in "$@"; do
  label="${spec%%:*}"; envs="${spec#*:}"
  env $envs timeout 300 python bench.py --steps ${AB_STEPS:-100} --no-extras ${AB_ARGS:-} 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; r=d['roofline']; print('$label', 'Gk/s %.2f'%(d['value']/1e9), 'ms %.4f'%d['ms_per_step'], 'w/r %.4f'%d['worst_over_random_time'], 'block %.1fus'%(1e3*k['block_sort']['avg_ms']), 'merge %.1fus'%(1e3*k['merge_pass']['avg_ms']), 'frac %.3f'%r['frac'], 'inreg %.1fus'%(1e3*r.get('merge_pass_in_region_est_ms',0)))" \
    >> gpurun_out/ab_env.txt 2>&1 || echo "$label failed" >> gpurun_out/ab_env.txt
done
