import sys, os, time, numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_spaa_berneys25_b200 as bcf, oracle, synthetic_inputs as si
dev = torch.device("cuda:0")
for n in [5000, 3840 * 2, 3840 * 2 + 1, 100003, 1 << 20, (1 << 24)]:
    x = si.uniform_u32(n, 7 + n)
    t0 = time.time()
    out = bcf.sort(torch.from_numpy(x.view(np.int32)).to(dev), params=bcf.make_params(15, 256))
    torch.cuda.synchronize()
    ok = np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(x))
    print(n, "ok" if ok else "MISMATCH", f"{time.time()-t0:.2f}s", flush=True)
