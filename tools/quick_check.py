"""Quick parity + timing check of the default sort on cuda:0 (one GPU session
step before the full test suite): sizes spanning 1..many merge passes, random
and worst-case, against the oracle; prints ms per sort."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402
import synthetic_inputs as si  # noqa: E402

dev = torch.device("cuda:0")
sizes = [int(x) for x in (sys.argv[1:] or ["100000", "1000003", str(1 << 24)])]
for n in sizes:
    for kind in ("random", "worst"):
        x = si.uniform_u32(n, 77 + n) if kind == "random" else bcf.worst_case_host(n, 31, 128, 5)
        t = torch.from_numpy(x.view(np.int32)).to(dev)
        out = bcf.sort(t)
        torch.cuda.synchronize()
        ok = np.array_equal(out.cpu().numpy().view(np.uint32), oracle.sort_u32(x))
        temp = bcf.temp_buffer(n, device=dev)
        for _ in range(3):
            bcf.sort(t, out=out, temp=temp)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(20):
            bcf.sort(t, out=out, temp=temp)
        torch.cuda.synchronize()
        ms = (time.perf_counter() - t0) / 20 * 1e3
        print(f"n={n} {kind}: parity={'OK' if ok else 'FAIL'} {ms:.3f} ms/sort  {n / ms / 1e6:.2f} G keys/s", flush=True)
