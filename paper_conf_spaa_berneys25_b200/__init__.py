"""paper_conf_spaa_berneys25_b200 -- B200-native bank-conflict-free mergesort.

Thin Python binding over the C ABI in include/bcf.h (libbcf.so, built
in-tree for sm_100a).  Argument marshalling only: every step of the sort runs
in the library's CUDA kernels.  PyTorch provides device memory and streams.
There is no CPU fallback: without the extension or without a CUDA tensor the
calls raise.

    sort(keys)                 u32 / i32 (as u32 bit patterns) / f32 (totalOrder)
    sort_pairs(keys, values)   stable by u32 key
    worst_case(n, E, u, seed)  Section 4 worst-case permutation (device tensor)
    worst_case_host(...)       same into a numpy array (no CUDA)
    merge(a, b)                stable merge of two sorted arrays (one CF merge pass)
    set_op(op, a, b)           union / intersection / difference / symmetric difference
    split_counts, merge_runs   distributed-sort phases (see dist.py)
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("BCF_LIB") or os.path.join(_HERE, "libbcf.so")  # BCF_LIB: A/B builds

BCF_SUCCESS = 0
BCF_ERROR_INVALID_VALUE = 1
BCF_ERROR_UNSUPPORTED = 2
BCF_ERROR_CUDA = 3
BCF_ERROR_TEMP_TOO_SMALL = 4
ALGO_CONFLICT_FREE = 0
ALGO_BASELINE = 1

# every symbol include/bcf.h declares
EXPORTED_SYMBOLS = [
    "bcf_default_params", "bcf_default_pairs_params", "bcf_sort_u32", "bcf_sort_f32", "bcf_sort_pairs_u32",
    "bcf_sort_u32_host_batch", "bcf_sort_plan", "bcf_worst_case_u32", "bcf_worst_case_u32_host", "bcf_split_counts_u32",
    "bcf_merge_runs_u32", "bcf_merge_u32", "bcf_status_string", "bcf_abi_version", "bcf_last_cuda_error",
    "bcf_profile_enable", "bcf_profile_collect", "bcf_launch_count", "bcf_debug_trace_copy", "bcf_set_op_u32",
    "bcf_merge_runs_ptrs_u32", "bcf_ipc_export", "bcf_ipc_open", "bcf_ipc_close",
]


class BcfError(RuntimeError):
    pass


class Params(ctypes.Structure):
    _fields_ = [("items_per_thread", ctypes.c_int32), ("block_threads", ctypes.c_int32),
                ("algo", ctypes.c_int32)]


class KernelStats(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 32), ("launches", ctypes.c_int64),
                ("total_ms", ctypes.c_double), ("keys", ctypes.c_uint64)]


_lib = None


def lib():
    """Load libbcf.so (raises if it was not built: run build() first)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise BcfError(f"{LIB_PATH} missing: build it with paper_conf_spaa_berneys25_b200.build.build()")
    L = ctypes.CDLL(LIB_PATH)
    vp, sz = ctypes.c_void_p, ctypes.c_size_t
    u64, i32 = ctypes.c_uint64, ctypes.c_int32
    P = ctypes.POINTER
    L.bcf_default_params.argtypes = [P(Params)]
    L.bcf_default_params.restype = None
    L.bcf_default_pairs_params.argtypes = [P(Params)]
    L.bcf_default_pairs_params.restype = None
    for name in ("bcf_sort_u32", "bcf_sort_f32"):
        f = getattr(L, name)
        f.argtypes = [vp, vp, u64, vp, P(sz), P(Params), vp]
        f.restype = ctypes.c_int
    L.bcf_sort_plan.argtypes = [u64, P(Params), i32, P(ctypes.c_int64), P(ctypes.c_int64), P(i32)]
    L.bcf_sort_plan.restype = ctypes.c_int
    L.bcf_sort_u32_host_batch.argtypes = [P(vp), P(vp), i32, u64, vp, P(sz), P(Params), vp]
    L.bcf_sort_u32_host_batch.restype = ctypes.c_int
    L.bcf_sort_pairs_u32.argtypes = [vp, vp, vp, vp, u64, vp, P(sz), P(Params), vp]
    L.bcf_sort_pairs_u32.restype = ctypes.c_int
    L.bcf_worst_case_u32.argtypes = [vp, u64, i32, i32, u64, vp]
    L.bcf_worst_case_u32.restype = ctypes.c_int
    L.bcf_worst_case_u32_host.argtypes = [vp, u64, i32, i32, u64]
    L.bcf_worst_case_u32_host.restype = ctypes.c_int
    L.bcf_split_counts_u32.argtypes = [vp, u64, vp, i32, vp, vp, vp]
    L.bcf_split_counts_u32.restype = ctypes.c_int
    L.bcf_merge_runs_u32.argtypes = [vp, vp, P(u64), i32, vp, vp, vp, P(sz), P(Params), vp]
    L.bcf_merge_runs_u32.restype = ctypes.c_int
    L.bcf_merge_u32.argtypes = [vp, u64, vp, u64, vp, vp, vp, vp, vp, P(sz), P(Params), vp]
    L.bcf_merge_u32.restype = ctypes.c_int
    L.bcf_status_string.argtypes = [ctypes.c_int]
    L.bcf_status_string.restype = ctypes.c_char_p
    L.bcf_abi_version.restype = i32
    L.bcf_last_cuda_error.restype = i32
    L.bcf_profile_enable.argtypes = [i32]
    L.bcf_profile_enable.restype = ctypes.c_int
    L.bcf_profile_collect.argtypes = [P(KernelStats), i32, P(i32)]
    L.bcf_profile_collect.restype = ctypes.c_int
    L.bcf_launch_count.restype = ctypes.c_int64
    L.bcf_merge_runs_ptrs_u32.argtypes = [vp, vp, i32, vp, vp, P(sz), P(Params), vp]
    L.bcf_merge_runs_ptrs_u32.restype = ctypes.c_int
    L.bcf_ipc_export.argtypes = [vp, vp, P(u64)]
    L.bcf_ipc_export.restype = ctypes.c_int
    L.bcf_ipc_open.argtypes = [vp, P(vp)]
    L.bcf_ipc_open.restype = ctypes.c_int
    L.bcf_ipc_close.argtypes = [vp]
    L.bcf_ipc_close.restype = ctypes.c_int
    L.bcf_set_op_u32.argtypes = [i32, vp, u64, vp, u64, vp, vp, vp, vp, P(ctypes.c_size_t), P(Params), vp]
    L.bcf_set_op_u32.restype = ctypes.c_int
    _lib = L
    return L


def _check(st: int, what: str):
    if st != BCF_SUCCESS:
        msg = lib().bcf_status_string(st).decode()
        if st == BCF_ERROR_CUDA:
            msg += f" (cudaError {lib().bcf_last_cuda_error()})"
        raise BcfError(f"{what}: {msg}")


def default_params() -> Params:
    p = Params()
    lib().bcf_default_params(ctypes.byref(p))
    return p


def default_pairs_params() -> Params:
    p = Params()
    lib().bcf_default_pairs_params(ctypes.byref(p))
    return p


def sort_plan(n: int, params: Params | None = None, pairs: bool = False) -> dict:
    """Pass plan of a sort (bcf_sort_plan): block-sort tile, merge tile, passes."""
    bt, mt, mp = ctypes.c_int64(0), ctypes.c_int64(0), ctypes.c_int32(0)
    pp = ctypes.byref(params) if params is not None else None
    _check(lib().bcf_sort_plan(n, pp, 1 if pairs else 0, ctypes.byref(bt), ctypes.byref(mt), ctypes.byref(mp)),
           "bcf_sort_plan")
    return {"block_sort_tile": bt.value, "merge_tile": mt.value, "merge_passes": mp.value}


def make_params(E: int = 0, u: int = 0, algo: int = ALGO_CONFLICT_FREE) -> Params:
    return Params(E, u, algo)


def _torch():
    import torch

    return torch


def _require_cuda(t, name):
    torch = _torch()
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise BcfError(f"{name} must be a CUDA tensor (no CPU path)")
    if not t.is_contiguous():
        raise BcfError(f"{name} must be contiguous")
    if t.element_size() != 4:
        raise BcfError(f"{name} must have 4-byte elements")


def _require_out(t, name, n, device):
    """An output tensor: CUDA, contiguous, 4-byte, n elements on `device`."""
    _require_cuda(t, name)
    if t.numel() != n:
        raise BcfError(f"{name} must hold {n} elements, has {t.numel()}")
    if t.device != device:
        raise BcfError(f"{name} is on {t.device}, expected {device}")


def _stream(t):
    torch = _torch()
    return ctypes.c_void_p(torch.cuda.current_stream(t.device).cuda_stream)


def _temp(nbytes: int, device):
    torch = _torch()
    return torch.empty(max(1, int(nbytes)), dtype=torch.uint8, device=device)


def temp_buffer(n: int, params: Params | None = None, pairs: bool = False, device="cuda"):
    """Temp storage for a sort of n keys (or pairs) with `params`, sized by the
    library's CUB-style query (d_temp = NULL)."""
    tb = ctypes.c_size_t(0)
    pp = ctypes.byref(params) if params is not None else None
    L = lib()
    if pairs:
        _check(L.bcf_sort_pairs_u32(None, None, None, None, n, None, ctypes.byref(tb), pp, None), "temp query")
    else:
        _check(L.bcf_sort_u32(None, None, n, None, ctypes.byref(tb), pp, None), "temp query")
    return _temp(tb.value, device)


def sort(keys, out=None, params: Params | None = None, temp=None):
    """Sort a 1-D CUDA tensor of 4-byte keys.  float32: IEEE totalOrder;
    int32 / uint32: keys are sorted as unsigned 32-bit bit patterns."""
    torch = _torch()
    _require_cuda(keys, "keys")
    n = keys.numel()
    if out is None:
        out = torch.empty_like(keys)
    _require_out(out, "out", n, keys.device)
    is_f32 = keys.dtype == torch.float32
    fn = lib().bcf_sort_f32 if is_f32 else lib().bcf_sort_u32
    tb = ctypes.c_size_t(0)
    pp = ctypes.byref(params) if params is not None else None
    _check(fn(None, None, n, None, ctypes.byref(tb), pp, None), "temp query")
    if temp is None or temp.numel() < tb.value:
        temp = _temp(tb.value, keys.device)
    tb = ctypes.c_size_t(temp.numel())
    with torch.cuda.device(keys.device):
        _check(fn(keys.data_ptr(), out.data_ptr(), n, temp.data_ptr(), ctypes.byref(tb), pp,
                  _stream(keys)), "bcf_sort")
    return out


def sort_pairs(keys, values, keys_out=None, values_out=None, params: Params | None = None, temp=None):
    torch = _torch()
    _require_cuda(keys, "keys")
    _require_cuda(values, "values")
    n = keys.numel()
    if values.numel() != n:
        raise BcfError("keys and values differ in length")
    if values.device != keys.device:
        raise BcfError("keys and values are on different devices")
    keys_out = torch.empty_like(keys) if keys_out is None else keys_out
    values_out = torch.empty_like(values) if values_out is None else values_out
    _require_out(keys_out, "keys_out", n, keys.device)
    _require_out(values_out, "values_out", n, keys.device)
    tb = ctypes.c_size_t(0)
    pp = ctypes.byref(params) if params is not None else None
    L = lib()
    _check(L.bcf_sort_pairs_u32(None, None, None, None, n, None, ctypes.byref(tb), pp, None), "temp query")
    if temp is None or temp.numel() < tb.value:
        temp = _temp(tb.value, keys.device)
    tb = ctypes.c_size_t(temp.numel())
    with torch.cuda.device(keys.device):
        _check(L.bcf_sort_pairs_u32(keys.data_ptr(), keys_out.data_ptr(), values.data_ptr(),
                                    values_out.data_ptr(), n, temp.data_ptr(), ctypes.byref(tb), pp,
                                    _stream(keys)), "bcf_sort_pairs_u32")
    return keys_out, values_out


def sort_host_batch(h_in, h_out, params: Params | None = None, temp=None, device="cuda"):
    """End-to-end sort of a batch of host (CPU) arrays of equal length n
    (bcf_sort_u32_host_batch): H2D, sort and D2H of consecutive arrays overlap.
    h_in / h_out: sequences of 1-D CPU tensors (pinned for async copies) of
    4-byte elements, sorted as u32 bit patterns.  Returns after the library's
    work is queued on the current stream of `device`; synchronise before
    reading h_out."""
    torch = _torch()
    if len(h_in) != len(h_out):
        raise BcfError("h_in and h_out differ in length")
    n = h_in[0].numel() if len(h_in) else 0
    for t in list(h_in) + list(h_out):
        if not isinstance(t, torch.Tensor) or t.is_cuda or t.element_size() != 4 or not t.is_contiguous() \
                or t.numel() != n:
            raise BcfError("h_in/h_out must be contiguous CPU tensors of n 4-byte elements")
    dev = torch.device(device)
    if dev.index is None:
        dev = torch.device("cuda", torch.cuda.current_device())
    L = lib()
    pp = ctypes.byref(params) if params is not None else None
    tb = ctypes.c_size_t(0)
    _check(L.bcf_sort_u32_host_batch(None, None, len(h_in), n, None, ctypes.byref(tb), pp, None), "temp query")
    if temp is None or temp.numel() < tb.value:
        temp = _temp(tb.value, dev)
    tb = ctypes.c_size_t(temp.numel())
    ins = (ctypes.c_void_p * max(1, len(h_in)))(*[t.data_ptr() for t in h_in])
    outs = (ctypes.c_void_p * max(1, len(h_out)))(*[t.data_ptr() for t in h_out])
    with torch.cuda.device(dev):
        _check(L.bcf_sort_u32_host_batch(ins, outs, len(h_in), n, temp.data_ptr(), ctypes.byref(tb), pp,
                                         ctypes.c_void_p(torch.cuda.current_stream(dev).cuda_stream)),
               "bcf_sort_u32_host_batch")
    return h_out


def worst_case(n: int, E: int, u: int, seed: int = 0, device="cuda"):
    torch = _torch()
    out = torch.empty(n, dtype=torch.int32, device=device)
    with torch.cuda.device(out.device):
        _check(lib().bcf_worst_case_u32(out.data_ptr() if n else None, n, E, u, seed & (2**64 - 1),
                                        _stream(out)), "bcf_worst_case_u32")
    return out


def worst_case_host(n: int, E: int, u: int, seed: int = 0) -> np.ndarray:
    out = np.empty(n, dtype=np.uint32)
    _check(lib().bcf_worst_case_u32_host(out.ctypes.data if n else None, n, E, u, seed & (2**64 - 1)),
           "bcf_worst_case_u32_host")
    return out


def split_counts(sorted_keys, pivots):
    """(lt, le) counts of each pivot in a sorted CUDA run (int64 tensors)."""
    torch = _torch()
    _require_cuda(sorted_keys, "sorted_keys")
    _require_cuda(pivots, "pivots")
    lt = torch.empty(pivots.numel(), dtype=torch.int64, device=sorted_keys.device)
    le = torch.empty_like(lt)
    with torch.cuda.device(sorted_keys.device):
        _check(lib().bcf_split_counts_u32(sorted_keys.data_ptr(), sorted_keys.numel(), pivots.data_ptr(),
                                          pivots.numel(), lt.data_ptr(), le.data_ptr(),
                                          _stream(sorted_keys)), "bcf_split_counts_u32")
    return lt, le


def merge_runs(runs, run_offsets, values=None, params: Params | None = None):
    """Stable merge of ascending runs stored back to back (run order breaks ties)."""
    torch = _torch()
    _require_cuda(runs, "runs")
    offs = np.ascontiguousarray(np.asarray(run_offsets, dtype=np.uint64))
    nruns = len(offs) - 1
    if nruns < 0 or int(offs[0]) != 0 or int(offs[-1]) != runs.numel() or np.any(np.diff(offs.astype(np.int64)) < 0):
        raise BcfError("run_offsets must start at 0, be non-decreasing and end at runs.numel()")
    if values is not None:
        _require_out(values, "values", runs.numel(), runs.device)
    out = torch.empty_like(runs)
    out_v = torch.empty_like(values) if values is not None else None
    L = lib()
    tb = ctypes.c_size_t(0)
    pp = ctypes.byref(params) if params is not None else None
    optr = offs.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))
    vptr = values.data_ptr() if values is not None else None
    _check(L.bcf_merge_runs_u32(runs.data_ptr(), vptr, optr, nruns, None, None, None, ctypes.byref(tb), pp,
                                None), "temp query")
    temp = _temp(tb.value, runs.device)
    tb = ctypes.c_size_t(temp.numel())
    with torch.cuda.device(runs.device):
        _check(L.bcf_merge_runs_u32(runs.data_ptr(), vptr, optr, nruns, out.data_ptr(),
                                    out_v.data_ptr() if out_v is not None else None, temp.data_ptr(),
                                    ctypes.byref(tb), pp, _stream(runs)), "bcf_merge_runs_u32")
    return (out, out_v) if values is not None else out


def merge_temp(na: int, nb: int, pairs: bool = False, params: Params | None = None, device="cuda"):
    """Temp storage for bcf_merge_u32 of na + nb keys (or pairs)."""
    tb = ctypes.c_size_t(0)
    pp = ctypes.byref(params) if params is not None else None
    vo = ctypes.c_void_p(16) if pairs else None  # only the pairs flag matters for the query
    _check(lib().bcf_merge_u32(None, na, None, nb, vo, vo, None, vo, None, ctypes.byref(tb), pp, None),
           "temp query")
    return _temp(tb.value, device)


def merge(a, b, a_values=None, b_values=None, params: Params | None = None, out=None, out_values=None,
          temp=None):
    """Stable merge of two ascending u32 arrays (ties: A first); values follow keys."""
    torch = _torch()
    _require_cuda(a, "a")
    _require_cuda(b, "b")
    if (a_values is None) != (b_values is None):
        raise ValueError("pass values for both inputs or for neither")
    if out is None:
        out = torch.empty(a.numel() + b.numel(), dtype=a.dtype, device=a.device)
    _require_cuda(out, "out")
    if out.numel() != a.numel() + b.numel():
        raise ValueError("out must hold a.numel() + b.numel() keys")
    if b.device != a.device:
        raise BcfError("a and b are on different devices")
    _require_out(out, "out", a.numel() + b.numel(), a.device)
    if a_values is not None:
        _require_out(a_values, "a_values", a.numel(), a.device)
        _require_out(b_values, "b_values", b.numel(), a.device)
        if out_values is None:
            out_values = torch.empty_like(out)
        _require_out(out_values, "out_values", out.numel(), a.device)
    L = lib()
    tb = ctypes.c_size_t(0)
    pp = ctypes.byref(params) if params is not None else None
    va = a_values.data_ptr() if a_values is not None else None
    vb = b_values.data_ptr() if b_values is not None else None
    vo = out_values.data_ptr() if a_values is not None else None
    _check(L.bcf_merge_u32(None, a.numel(), None, b.numel(), va, vb, None, vo, None, ctypes.byref(tb), pp, None),
           "temp query")
    if temp is None or temp.numel() < tb.value:
        temp = _temp(tb.value, a.device)
    tb = ctypes.c_size_t(temp.numel())
    with torch.cuda.device(a.device):
        _check(L.bcf_merge_u32(a.data_ptr(), a.numel(), b.data_ptr(), b.numel(), va, vb, out.data_ptr(), vo,
                               temp.data_ptr(), ctypes.byref(tb), pp, _stream(a)), "bcf_merge_u32")
    return (out, out_values) if a_values is not None else out


def merge_runs_ptrs(run_ptrs, run_lens, device, dtype=None, params: Params | None = None, out=None):
    """bcf_merge_runs_ptrs_u32: stable merge of sorted runs given as raw
    device pointers (ints; local or peer-mapped) and lengths; returns a new
    CUDA tensor on `device` (int32 unless dtype is given)."""
    torch = _torch()
    nr = len(run_ptrs)
    if len(run_lens) != nr:
        raise BcfError("run_ptrs and run_lens differ in length")
    n = int(sum(int(x) for x in run_lens))
    if out is None:
        out = torch.empty(max(1, n), dtype=dtype or torch.int32, device=device)
    _require_cuda(out, "out")
    ptrs = (ctypes.c_void_p * max(1, nr))(*[int(p) for p in run_ptrs])
    lens = (ctypes.c_uint64 * max(1, nr))(*[int(x) for x in run_lens])
    L = lib()
    pp = ctypes.byref(params) if params is not None else None
    tb = ctypes.c_size_t(0)
    _check(L.bcf_merge_runs_ptrs_u32(ptrs, lens, nr, None, None, ctypes.byref(tb), pp, None), "temp query")
    temp = _temp(tb.value, out.device)
    tb = ctypes.c_size_t(temp.numel())
    with torch.cuda.device(out.device):
        _check(L.bcf_merge_runs_ptrs_u32(ptrs, lens, nr, out.data_ptr(), temp.data_ptr(), ctypes.byref(tb), pp,
                                         _stream(out)), "bcf_merge_runs_ptrs_u32")
    return out[:n]


def ipc_export(t) -> tuple:
    """(handle bytes, byte offset of t's data in its allocation)."""
    _require_cuda(t, "t")
    h = ctypes.create_string_buffer(64)
    off = ctypes.c_uint64(0)
    _check(lib().bcf_ipc_export(t.data_ptr(), h, ctypes.byref(off)), "bcf_ipc_export")
    return bytes(h.raw), int(off.value)


def ipc_open(handle: bytes) -> int:
    base = ctypes.c_void_p(0)
    _check(lib().bcf_ipc_open(ctypes.create_string_buffer(handle, 64), ctypes.byref(base)), "bcf_ipc_open")
    return int(base.value)


def ipc_close(base: int):
    _check(lib().bcf_ipc_close(ctypes.c_void_p(base)), "bcf_ipc_close")


SET_OPS = {"union": 0, "intersection": 1, "difference": 2, "symmetric_difference": 3}


def set_op(op: str, a, b, with_source: bool = False, params: Params | None = None):
    """Set operation of two ascending 1-D CUDA tensors of 4-byte keys (u32
    order), multiset semantics of std::set_* (bcf_set_op_u32).  Returns the
    kept keys (and, with_source, the int32 tags: A index or 0x80000000 | B
    index).  Reads the output count back (synchronises the stream)."""
    torch = _torch()
    _require_cuda(a, "a")
    _require_cuda(b, "b")
    if b.device != a.device:
        raise BcfError("a and b are on different devices")
    if op not in SET_OPS:
        raise BcfError(f"unknown set operation {op!r}")
    n = a.numel() + b.numel()
    out = torch.empty(max(1, n), dtype=a.dtype, device=a.device)
    src = torch.empty(max(1, n), dtype=torch.int32, device=a.device) if with_source else None
    cnt = torch.zeros(1, dtype=torch.int64, device=a.device)
    L = lib()
    pp = ctypes.byref(params) if params is not None else None
    tb = ctypes.c_size_t(0)
    _check(L.bcf_set_op_u32(SET_OPS[op], None, a.numel(), None, b.numel(), None, None, None, None,
                            ctypes.byref(tb), pp, None), "temp query")
    temp = _temp(tb.value, a.device)
    tb = ctypes.c_size_t(temp.numel())
    with torch.cuda.device(a.device):
        _check(L.bcf_set_op_u32(SET_OPS[op], a.data_ptr() if a.numel() else None, a.numel(),
                                b.data_ptr() if b.numel() else None, b.numel(), out.data_ptr(),
                                src.data_ptr() if src is not None else None, cnt.data_ptr(), temp.data_ptr(),
                                ctypes.byref(tb), pp, _stream(a)), "bcf_set_op_u32")
    k = int(cnt.item())
    return (out[:k], src[:k]) if with_source else out[:k]


def profile_enable(on: bool = True):
    _check(lib().bcf_profile_enable(1 if on else 0), "bcf_profile_enable")


def profile_collect() -> dict:
    arr = (KernelStats * 32)()
    cnt = ctypes.c_int32(0)
    _check(lib().bcf_profile_collect(arr, 32, ctypes.byref(cnt)), "bcf_profile_collect")
    return {arr[i].name.decode(): {"launches": arr[i].launches, "total_ms": arr[i].total_ms,
                                   "keys": arr[i].keys} for i in range(cnt.value)}


def launch_count() -> int:
    return int(lib().bcf_launch_count())


def abi_version() -> int:
    return int(lib().bcf_abi_version())
