"""Per-kernel times (library event profiler) of bcf_set_op_u32 on two sorted 2^L u32 arrays
over 2^(L+1) values (the bench's set-operation leg).  usage: time_setop.py [L] [op]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_spaa_berneys25_b200 as bcf
L = int(sys.argv[1]) if len(sys.argv) > 1 else 25
op = sys.argv[2] if len(sys.argv) > 2 else "intersection"
g = torch.Generator(device="cuda").manual_seed(3)
a = torch.randint(0, 1 << (L + 1), (1 << L,), dtype=torch.int32, device="cuda", generator=g).sort()[0]
b = torch.randint(0, 1 << (L + 1), (1 << L,), dtype=torch.int32, device="cuda", generator=g).sort()[0]
for _ in range(3):
    bcf.set_op(op, a, b)
torch.cuda.synchronize()
bcf.profile_enable(True)
for _ in range(10):
    bcf.set_op(op, a, b)
torch.cuda.synchronize()
st = bcf.profile_collect()
bcf.profile_enable(False)
print(op, {k: "%.1f us x %d" % (1e3 * v["total_ms"] / v["launches"], v["launches"] // 10) for k, v in st.items()})
