"""A/B: stable pairs sort at 2^26 (BASELINE configs[2]), median of 10, L2 flushed;
run with and without BCF_PAIRS_TMA=1 (window vs exact-split TMA merge passes)."""
import json, os, sys
import torch
sys.path.insert(0, os.getcwd())
import paper_conf_spaa_berneys25_b200 as bcf, synthetic_inputs as si
dev = torch.device("cuda:0"); n = 1 << 26
k = si.dup_u32_torch(n, si.config_seed(4), dev); v = si.iota_u32_torch(n, dev)
ko, vo = torch.empty_like(k), torch.empty_like(v)
prm = bcf.default_pairs_params(); temp = bcf.temp_buffer(n, prm, pairs=True, device=dev)
flush = torch.empty(64 << 20, dtype=torch.int32, device=dev)
for _ in range(3): bcf.sort_pairs(k, v, ko, vo, params=prm, temp=temp)
torch.cuda.synchronize(); ts = []
for i in range(10):
    flush.fill_(i); a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record(); bcf.sort_pairs(k, v, ko, vo, params=prm, temp=temp); b.record(); torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
ts.sort()
print(json.dumps({"pairs_tma_forced": os.environ.get("BCF_PAIRS_TMA", "0"), "median_ms": ts[5], "pairs_per_s": n / (ts[5] / 1e3)}))
