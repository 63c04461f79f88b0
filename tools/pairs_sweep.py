"""Time the stable pairs sort (2^26 u32 pairs, configs[2]) for several (E, u)."""
import os, sys, json
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_spaa_berneys25_b200 as bcf, synthetic_inputs as si

dev = torch.device("cuda:0")
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 26
cfgs = sys.argv[2].split(",") if len(sys.argv) > 2 else ["31:128", "15:256", "17:256", "15:128", "17:128", "16:256", "13:256", "11:256", "9:256"]
k = si.dup_u32_torch(n, si.config_seed(4), dev)
v = si.iota_u32_torch(n, dev)
ko, vo = torch.empty_like(k), torch.empty_like(v)
flush = torch.empty(64 << 20, dtype=torch.int32, device=dev)
for c in cfgs:
    E, u = map(int, c.split(":"))
    p = bcf.make_params(E, u, 0)
    try:
        temp = bcf.temp_buffer(n, p, pairs=True, device=dev)
        for _ in range(2):
            bcf.sort_pairs(k, v, ko, vo, params=p, temp=temp)
        torch.cuda.synchronize()
        ts = []
        for i in range(5):
            flush.fill_(i)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); bcf.sort_pairs(k, v, ko, vo, params=p, temp=temp); b.record()
            torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
        bcf.profile_enable(True)
        bcf.sort_pairs(k, v, ko, vo, params=p, temp=temp)
        torch.cuda.synchronize()
        bcf.profile_enable(False)
        pr = bcf.profile_collect()
        ms = min(ts)
        print(json.dumps({"E": E, "u": u, "ms": ms, "Gpairs_s": n / ms / 1e6,
                          "block_ms": pr["block_sort"]["total_ms"], "merge_avg_ms": pr["merge_pass"]["total_ms"] / pr["merge_pass"]["launches"],
                          "merge_launches": pr["merge_pass"]["launches"]}))
        del temp
    except Exception as e:  # noqa: BLE001
        print(json.dumps({"E": E, "u": u, "error": str(e)}))
    sys.stdout.flush()
