set +e
mkdir -p gpurun_out
for ln in 24 27; do
for cfg in 31_128 15_128 15_256 17_128 17_256 13_256 11_256 9_256 15_512 31_256; do
  set -- ${cfg//_/ }
  timeout 300 python bench.py --E $1 --u $2 --log2n $ln --steps 40 --no-extras 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('n 2^$ln E',d['config']['E'],'u',d['config']['u'],'P',d['config']['merge_passes'],'Gk/s %.2f'%(d['value']/1e9),'w/r %.4f'%d['worst_over_random_time'],'block %.1fus'%(1e3*k['block_sort']['avg_ms']),'merge %.1fus'%(1e3*k['merge_pass']['avg_ms']),'frac %.3f'%d['roofline']['frac'])"
done; done > gpurun_out/qb.txt 2>&1
BCF_NO_TMA=1 timeout 300 python bench.py --steps 40 --no-extras | tail -1 > gpurun_out/qb_notma.json
