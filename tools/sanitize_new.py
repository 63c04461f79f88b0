"""Small invocations of the round-2 kernels for compute-sanitizer (memcheck /
racecheck): the even-E window merge pass (keys, pairs), the multi-pass launch,
set operations, the device worst-case generator and merge_runs_ptrs with local
pointers; every result checked against the oracle."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402
import synthetic_inputs as si  # noqa: E402
from oracle import worstcase as wc  # noqa: E402

dev = torch.device("cuda:0")


def d(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.uint32).view(np.int32).copy()).to(dev)


def h(t):
    return t.cpu().numpy().view(np.uint32)


n = 70001
x = si.uniform_u32(n, 3) & np.uint32(0xFFFF)
for E, u in [(16, 128), (12, 256), (8, 512), (10, 128), (14, 256)]:
    p = bcf.make_params(E, u)
    assert np.array_equal(h(bcf.sort(d(x), params=p)), oracle.sort_u32(x)), (E, u)
    ko, vo = bcf.sort_pairs(d(x), d(np.arange(n, dtype=np.uint32)), params=p)
    ek, ev = oracle.sort_pairs_u32(x, np.arange(n, dtype=np.uint32))
    assert np.array_equal(h(ko), ek) and np.array_equal(h(vo), ev), (E, u, "pairs")
for op in ("union", "intersection", "difference", "symmetric_difference"):
    a, b = np.sort(x[:40000]), np.sort(x[40000:])
    k, s = bcf.set_op(op, d(a), d(b), with_source=True)
    ek, es = oracle.set_op_u32(op, a, b)
    assert np.array_equal(h(k), ek) and np.array_equal(h(s), es), op
w = bcf.worst_case(50000, 31, 128, seed=9, device=dev)
assert np.array_equal(h(w), wc.worst_case_input(50000, 31, 128, 9))
runs = [np.sort(si.uniform_u32(m, 10 + m)) for m in (1000, 0, 3333, 17)]
ts = [d(r) for r in runs]
out = bcf.merge_runs_ptrs([t.data_ptr() for t in ts], [r.size for r in runs], dev)
assert np.array_equal(h(out), oracle.sort_u32(np.concatenate(runs)))
torch.cuda.synchronize()
print("sanitize_new ok")
