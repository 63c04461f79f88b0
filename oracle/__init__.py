"""oracle -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously correct CPU implementation of what the CUDA path of
paper_conf_spaa_berneys25_b200 computes, written from the paper
(/root/reference/PAPER.md, cited as PAPER.md:<line>):

    sort_oracle.c   stable top-down mergesort: u32, f32 (IEEE totalOrder), pairs
    addrmap.py      pi, rho and Alg. 1's gather schedule (§3)
    dmm.py          DMM bank-conflict cost model + Thrust serial-merge address stream
    worstcase.py    Section 4 worst-case construction (S, T, Theorem 8) + composition
    setops_oracle.c set union / intersection / difference / symmetric difference
                    of two sorted sequences, multiset semantics of ISO C++
                    [alg.set.operations] (the paper's "parallel scan of a pair of
                    arrays")
    cpu_baselines.cpp  std::stable_sort (1 core) and a std::thread parallel
                    stable mergesort (all cores): the further CPU baselines of
                    SURVEY.md §8(d), also a library cross-check of the oracle

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` leg may import, call, link or execute anything under
oracle/.  The product path never does, and the oracle never imports the
product package: the two share only `synthetic_inputs` (seeded generators,
none of the method's arithmetic).

Parity status of each function is listed in DESIGN.md §"Oracle and pins"; every
function here is pinned by tests/test_oracle_*.py to something other than
itself (library routines, brute force, the paper's figures and closed forms).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sort_oracle.c")
_SRC_SET = os.path.join(_HERE, "setops_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


_CPP_SRC = os.path.join(_HERE, "cpu_baselines.cpp")
_CPP_LIB = os.path.join(_HERE, "libcpu_baselines.so")
_cpp = None


def build(force: bool = False) -> str:
    """Compile sort_oracle.c with gcc (plain C, -O2, single thread) and the
    CPU baselines with g++ (-O2, std::thread)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(os.path.getmtime(_SRC),
                                                                           os.path.getmtime(_SRC_SET)):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c99", "-shared", "-fPIC", "-o", _LIB, _SRC, _SRC_SET]
        )
    if force or not os.path.exists(_CPP_LIB) or os.path.getmtime(_CPP_LIB) < os.path.getmtime(_CPP_SRC):
        subprocess.check_call(
            ["g++", "-O2", "-std=c++17", "-pthread", "-shared", "-fPIC", "-o", _CPP_LIB, _CPP_SRC]
        )
    return _LIB


def cpp_lib():
    global _cpp
    if _cpp is None:
        build()
        L = ctypes.CDLL(_CPP_LIB)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        L.baseline_std_stable_sort_u32.argtypes = [u32p, u32p, ctypes.c_uint64]
        L.baseline_std_stable_sort_u32.restype = ctypes.c_int
        L.baseline_parallel_mergesort_u32.argtypes = [u32p, u32p, ctypes.c_uint64, ctypes.c_int]
        L.baseline_parallel_mergesort_u32.restype = ctypes.c_int
        _cpp = L
    return _cpp


def std_stable_sort_u32(keys: np.ndarray) -> np.ndarray:
    """CPU baseline (ii): std::stable_sort on one core."""
    k = np.ascontiguousarray(keys, dtype=np.uint32)
    out = np.empty_like(k)
    cpp_lib().baseline_std_stable_sort_u32(_p(k), _p(out), k.size)
    return out


def parallel_mergesort_u32(keys: np.ndarray, threads: int) -> np.ndarray:
    """CPU baseline (iii): chunked std::stable_sort + parallel std::merge tree."""
    k = np.ascontiguousarray(keys, dtype=np.uint32)
    out = np.empty_like(k)
    cpp_lib().baseline_parallel_mergesort_u32(_p(k), _p(out), k.size, int(threads))
    return out


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        for name in ("oracle_sort_u32", "oracle_sort_f32"):
            f = getattr(L, name)
            f.argtypes = [u32p, u32p, ctypes.c_uint64]
            f.restype = ctypes.c_int
        L.oracle_sort_pairs_u32.argtypes = [u32p, u32p, u32p, u32p, ctypes.c_uint64]
        L.oracle_sort_pairs_u32.restype = ctypes.c_int
        L.oracle_set_op_u32.argtypes = [ctypes.c_int, u32p, ctypes.c_uint64, u32p, ctypes.c_uint64, u32p, u32p,
                                         ctypes.POINTER(ctypes.c_uint64)]
        L.oracle_set_op_u32.restype = ctypes.c_int
        L.oracle_f32_total_less.argtypes = [ctypes.c_uint32, ctypes.c_uint32]
        L.oracle_f32_total_less.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


def sort_u32(keys: np.ndarray) -> np.ndarray:
    k = np.ascontiguousarray(keys, dtype=np.uint32)
    out = np.empty_like(k)
    if lib().oracle_sort_u32(_p(k), _p(out), k.size) != 0:
        raise MemoryError("oracle_sort_u32")
    return out


def sort_f32_bits(bits: np.ndarray) -> np.ndarray:
    """Keys given and returned as uint32 bit patterns of binary32 floats."""
    k = np.ascontiguousarray(bits, dtype=np.uint32)
    out = np.empty_like(k)
    if lib().oracle_sort_f32(_p(k), _p(out), k.size) != 0:
        raise MemoryError("oracle_sort_f32")
    return out


def sort_pairs_u32(keys: np.ndarray, vals: np.ndarray):
    k = np.ascontiguousarray(keys, dtype=np.uint32)
    v = np.ascontiguousarray(vals, dtype=np.uint32)
    assert k.size == v.size
    ko = np.empty_like(k)
    vo = np.empty_like(v)
    if lib().oracle_sort_pairs_u32(_p(k), _p(v), _p(ko), _p(vo), k.size) != 0:
        raise MemoryError("oracle_sort_pairs_u32")
    return ko, vo


SET_OPS = {"union": 0, "intersection": 1, "difference": 2, "symmetric_difference": 3}


def set_op_u32(op: str, a: np.ndarray, b: np.ndarray):
    """(keys, sources) of the set operation `op` on ascending a and b
    (setops_oracle.c; source = A index, or 0x80000000 | B index)."""
    a = np.ascontiguousarray(a, dtype=np.uint32)
    b = np.ascontiguousarray(b, dtype=np.uint32)
    out = np.empty(a.size + b.size + 1, dtype=np.uint32)
    src = np.empty_like(out)
    cnt = ctypes.c_uint64(0)
    if lib().oracle_set_op_u32(SET_OPS[op], _p(a), a.size, _p(b), b.size, _p(out), _p(src), ctypes.byref(cnt)) != 0:
        raise ValueError(op)
    return out[:cnt.value].copy(), src[:cnt.value].copy()


def f32_total_less(a: int, b: int) -> bool:
    return bool(lib().oracle_f32_total_less(a & 0xFFFFFFFF, b & 0xFFFFFFFF))


def dist_rank_slice(sorted_global: np.ndarray, rank: int, world: int):
    """Rank r of an exactly balanced distributed sort holds positions
    [floor(r n / p), floor((r+1) n / p)) of the global stable order."""
    n = sorted_global.shape[0]
    return sorted_global[(rank * n) // world:((rank + 1) * n) // world]
