"""Per-pass timeline of the multi-pass merge launch (BCF_TRACE_MULTI=1):
for each pass p >= 1 the spread over CTAs of wait start / inputs ready /
published, relative to the earliest timestamp, and the mean wait."""
import ctypes
import os
import sys

os.environ["BCF_TRACE_MULTI"] = "1"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402
import synthetic_inputs as si  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 24
dev = torch.device("cuda:0")
x = si.uniform_u32_torch(n, 99, dev)
out = torch.empty_like(x)
temp = bcf.temp_buffer(n, device=dev)
for _ in range(3):
    bcf.sort(x, out=out, temp=temp)
torch.cuda.synchronize()
plan = bcf.sort_plan(n)
P = plan["merge_passes"]
G = 740
buf = np.zeros(2048 * 256, dtype=np.uint64)
L = bcf.lib()
L.bcf_debug_trace_copy.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
L.bcf_debug_trace_copy.restype = ctypes.c_int
st = L.bcf_debug_trace_copy(ctypes.c_void_p(buf.ctypes.data), buf.nbytes)
assert st == 0, st
tr = buf.reshape(2048, 256)[:G].astype(np.int64)
valid = tr[:, 2] > 0
t0 = tr[valid][:, [4 * p + k for p in range(P) for k in range(3)]]
t0 = t0[t0 > 0].min()
print(f"n={n} passes={P} ctas={valid.sum()}")
print("pass  wait_start(min/p50/max)   ready(min/p50/max)    published(min/p50/max)   mean_wait_us")
for p in range(P):
    ws = tr[valid, 4 * p] if p > 0 else None
    rd = tr[valid, 4 * p + 1] if p > 0 else None
    pb = tr[valid, 4 * p + 2]
    f = lambda a: "%7.1f %7.1f %7.1f" % tuple((np.percentile(a, q) - t0) / 1e3 for q in (0, 50, 100))  # noqa: E731
    if p == 0:
        print(f"{p:4d}  {'-':>23s}   {'-':>23s}   {f(pb)}")
    else:
        print(f"{p:4d}  {f(ws)}   {f(rd)}   {f(pb)}   {np.mean(rd - ws) / 1e3:7.2f}")
