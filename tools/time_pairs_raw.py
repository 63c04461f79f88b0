"""Pairs merge-pass timing through a bare ctypes load of any libbcf build (A/B of
older commits whose ABI lacks later entry points).  usage: time_pairs_raw.py LIB [log2n]"""
import ctypes, sys
import torch
L = ctypes.CDLL(sys.argv[1])
n = 1 << (int(sys.argv[2]) if len(sys.argv) > 2 else 26)
g = torch.Generator(device="cuda").manual_seed(1)
k = torch.randint(0, 1 << 16, (n,), dtype=torch.int32, device="cuda", generator=g)
v = torch.arange(n, dtype=torch.int32, device="cuda")
ko, vo = torch.empty_like(k), torch.empty_like(v)
tb = ctypes.c_size_t(0)
vp = ctypes.c_void_p
L.bcf_sort_pairs_u32.argtypes = [vp, vp, vp, vp, ctypes.c_uint64, vp, ctypes.POINTER(ctypes.c_size_t), vp, vp]
assert L.bcf_sort_pairs_u32(k.data_ptr(), ko.data_ptr(), v.data_ptr(), vo.data_ptr(), n, None, ctypes.byref(tb), None, None) == 0
tmp = torch.empty(tb.value, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream().cuda_stream
def run():
    assert L.bcf_sort_pairs_u32(k.data_ptr(), ko.data_ptr(), v.data_ptr(), vo.data_ptr(), n, tmp.data_ptr(),
                                ctypes.byref(tb), None, vp(s)) == 0
for _ in range(3):
    run()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    run()
e1.record()
torch.cuda.synchronize()
print(sys.argv[1], "pairs sort ms %.3f" % (e0.elapsed_time(e1) / 10))
