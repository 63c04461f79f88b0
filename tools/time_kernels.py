"""Per-kernel average launch times (library CUDA-event profiler) of a 2^L u32 sort
(or a stable pairs sort with the third argument "pairs": keys & 0xFFFF, values = index).
usage: python tools/time_kernels.py [log2n] [reps] [pairs]   (BCF_LIB selects a variant build)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_spaa_berneys25_b200 as bcf
import synthetic_inputs as si
L = int(sys.argv[1]) if len(sys.argv) > 1 else 24
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
pairs = len(sys.argv) > 3 and sys.argv[3] == "pairs"
x = si.uniform_u32_torch(1 << L, si.config_seed(1), torch.device("cuda:0"))
if pairs:
    x = x & 0xFFFF
    v = torch.arange(1 << L, dtype=torch.int32, device=x.device)
run = (lambda: bcf.sort_pairs(x, v)) if pairs else (lambda: bcf.sort(x))
for _ in range(3):
    run()
torch.cuda.synchronize()
bcf.profile_enable(True)
for _ in range(reps):
    run()
torch.cuda.synchronize()
st = bcf.profile_collect()
bcf.profile_enable(False)
print(os.environ.get("BCF_LIB", "default"), {k: "%.1f us x %d" % (1e3 * v["total_ms"] / v["launches"], v["launches"] // reps)
                                            for k, v in st.items()})
