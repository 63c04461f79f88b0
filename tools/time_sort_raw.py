"""Keys-sort timing through a bare ctypes load of any libbcf build (cross-commit A/B),
with the library's per-kernel event profiler.  usage: time_sort_raw.py LIB [log2n] [E u algo]"""
import ctypes, sys
import torch
L = ctypes.CDLL(sys.argv[1])
n = 1 << (int(sys.argv[2]) if len(sys.argv) > 2 else 24)
g = torch.Generator(device="cuda").manual_seed(1)
k = torch.randint(-2**31, 2**31 - 1, (n,), dtype=torch.int32, device="cuda", generator=g)
ko = torch.empty_like(k)
tb = ctypes.c_size_t(0)
vp = ctypes.c_void_p


class Params(ctypes.Structure):
    _fields_ = [("items_per_thread", ctypes.c_int32), ("block_threads", ctypes.c_int32), ("algo", ctypes.c_int32)]


prm = Params(*[int(a) for a in sys.argv[3:6]]) if len(sys.argv) > 5 else None
pp = ctypes.byref(prm) if prm is not None else None
L.bcf_sort_u32.argtypes = [vp, vp, ctypes.c_uint64, vp, ctypes.POINTER(ctypes.c_size_t), vp, vp]
assert L.bcf_sort_u32(k.data_ptr(), ko.data_ptr(), n, None, ctypes.byref(tb), pp, None) == 0
tmp = torch.empty(tb.value, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream().cuda_stream
def run():
    assert L.bcf_sort_u32(k.data_ptr(), ko.data_ptr(), n, tmp.data_ptr(), ctypes.byref(tb), pp, vp(s)) == 0
for _ in range(3):
    run()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20):
    run()
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 20


class KS(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 32), ("launches", ctypes.c_int64), ("total_ms", ctypes.c_double),
                ("keys", ctypes.c_uint64)]


L.bcf_profile_enable(1)
for _ in range(20):
    run()
torch.cuda.synchronize()
arr = (KS * 32)()
cnt = ctypes.c_int32(0)
L.bcf_profile_collect(arr, 32, ctypes.byref(cnt))
st = {arr[i].name.decode(): "%.1f us" % (1e3 * arr[i].total_ms / arr[i].launches) for i in range(cnt.value)}
print(sys.argv[1], sys.argv[3:6], "sort ms %.4f" % ms, st)
