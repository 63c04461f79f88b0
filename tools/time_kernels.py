"""Per-kernel average launch times (library CUDA-event profiler) of a 2^L u32 sort.
usage: python tools/time_kernels.py [log2n] [reps]   (BCF_LIB selects a variant build)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_spaa_berneys25_b200 as bcf
import synthetic_inputs as si
L = int(sys.argv[1]) if len(sys.argv) > 1 else 24
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
x = si.uniform_u32_torch(1 << L, si.config_seed(1), torch.device("cuda:0"))
for _ in range(3):
    bcf.sort(x)
torch.cuda.synchronize()
bcf.profile_enable(True)
for _ in range(reps):
    bcf.sort(x)
torch.cuda.synchronize()
st = bcf.profile_collect()
bcf.profile_enable(False)
print(os.environ.get("BCF_LIB", "default"), {k: "%.1f us x %d" % (1e3 * v["total_ms"] / v["launches"], v["launches"] // reps)
                                            for k, v in st.items()})
