import os, sys, json, numpy as np, torch
sys.path.insert(0, os.getcwd())
import paper_conf_spaa_berneys25_b200 as bcf, synthetic_inputs as si
dev = torch.device("cuda:0"); n = 1 << 26
rk = torch.cat([bcf.sort(si.uniform_u32_torch(n // 8, si.config_seed(6), dev, lo=r * (n // 8))) for r in range(8)])
offs = np.arange(9, dtype=np.uint64) * np.uint64(n // 8)
flush = torch.empty(64 << 20, dtype=torch.int32, device=dev)
for _ in range(3): bcf.merge_runs(rk, offs)
torch.cuda.synchronize(); ts = []
for i in range(20):
    flush.fill_(i); a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record(); bcf.merge_runs(rk, offs); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
ts.sort(); print(json.dumps({"no_tma": os.environ.get("BCF_NO_TMA", "0"), "median_ms": ts[10], "gbs_3x8B": 24 * n / (ts[10] / 1e3) / 1e9}))
