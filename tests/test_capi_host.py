"""CPU-side checks of the C ABI: the library loads, exports every symbol
include/bcf.h declares, validates arguments synchronously, and its host-side
worst-case generator matches the oracle's construction bit for bit.  No
compute call touches a GPU here."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_spaa_berneys25_b200 as bcf
from paper_conf_spaa_berneys25_b200 import build as bcf_build
from oracle import worstcase as wc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    bcf_build.build()


def header_symbols():
    src = open(os.path.join(ROOT, "include", "bcf.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bcf_[a-z0-9_]+)\s*\(", src)))


def test_every_declared_symbol_is_exported():
    syms = header_symbols()
    assert len(syms) >= 14
    L = bcf.lib()
    for s in syms:
        assert hasattr(L, s), s
    assert sorted(bcf.EXPORTED_SYMBOLS) == syms


def test_abi_version_and_status_strings():
    assert bcf.abi_version() == 1
    L = bcf.lib()
    for code, name in [(0, "BCF_SUCCESS"), (1, "BCF_ERROR_INVALID_VALUE"), (2, "BCF_ERROR_UNSUPPORTED"),
                       (3, "BCF_ERROR_CUDA"), (4, "BCF_ERROR_TEMP_TOO_SMALL")]:
        assert L.bcf_status_string(code).decode() == name


def test_default_params():
    import bench

    p = bcf.default_params()
    assert (p.items_per_thread, p.block_threads) == (bench.DEFAULT_E, bench.DEFAULT_U)
    assert 7 <= p.items_per_thread <= 17 or p.items_per_thread == 31
    assert p.block_threads in (128, 256, 512)
    assert p.algo == bcf.ALGO_CONFLICT_FREE
    q = bcf.default_pairs_params()
    assert (q.items_per_thread, q.block_threads, q.algo) == (11, 256, bcf.ALGO_CONFLICT_FREE)


def _query(fn, n, params=None, pairs=False):
    tb = ctypes.c_size_t(0)
    pp = ctypes.byref(params) if params is not None else None
    if pairs:
        st = fn(None, None, None, None, n, None, ctypes.byref(tb), pp, None)
    else:
        st = fn(None, None, n, None, ctypes.byref(tb), pp, None)
    return st, tb.value


def test_temp_query_and_validation():
    L = bcf.lib()
    for n in [0, 1, 1000, 1 << 24]:
        st, tb = _query(L.bcf_sort_u32, n)
        assert st == 0 and tb >= 4 * n
        st, tbp = _query(L.bcf_sort_pairs_u32, n, pairs=True)
        assert st == 0 and tbp >= 8 * n
    # unsupported parameters are rejected before any launch
    assert _query(L.bcf_sort_u32, 100, bcf.make_params(6, 256))[0] == bcf.BCF_ERROR_UNSUPPORTED
    assert _query(L.bcf_sort_u32, 100, bcf.make_params(18, 256))[0] == bcf.BCF_ERROR_UNSUPPORTED
    assert _query(L.bcf_sort_u32, 100, bcf.make_params(30, 256))[0] == bcf.BCF_ERROR_UNSUPPORTED
    assert _query(L.bcf_sort_u32, 100, bcf.make_params(32, 256))[0] == bcf.BCF_ERROR_UNSUPPORTED
    assert _query(L.bcf_sort_u32, 100, bcf.make_params(31, 128))[0] == 0
    assert _query(L.bcf_sort_u32, 100, bcf.make_params(15, 384))[0] == bcf.BCF_ERROR_UNSUPPORTED
    assert _query(L.bcf_sort_u32, 100, bcf.make_params(15, 256, 7))[0] == bcf.BCF_ERROR_INVALID_VALUE
    assert _query(L.bcf_sort_pairs_u32, 100, bcf.make_params(15, 256, bcf.ALGO_BASELINE),
                  pairs=True)[0] == bcf.BCF_ERROR_UNSUPPORTED
    # NULL temp_bytes
    assert L.bcf_sort_u32(None, None, 10, None, None, None, None) == bcf.BCF_ERROR_INVALID_VALUE
    # temp too small / null data pointers are reported synchronously
    tb = ctypes.c_size_t(16)
    assert L.bcf_sort_u32(None, None, 1000, ctypes.c_void_p(256), ctypes.byref(tb), None,
                          None) == bcf.BCF_ERROR_TEMP_TOO_SMALL
    _, need = _query(L.bcf_sort_u32, 1000)
    tb = ctypes.c_size_t(need)
    assert L.bcf_sort_u32(None, None, 1000, ctypes.c_void_p(256), ctypes.byref(tb), None,
                          None) == bcf.BCF_ERROR_INVALID_VALUE
    # n = 0 is a no-op
    tb = ctypes.c_size_t(need)
    assert L.bcf_sort_u32(None, None, 0, ctypes.c_void_p(256), ctypes.byref(tb), None, None) == 0
    # worst-case generator argument checks
    assert L.bcf_worst_case_u32_host(None, 10, 15, 256, 0) == bcf.BCF_ERROR_INVALID_VALUE
    out = np.empty(10, np.uint32)
    assert L.bcf_worst_case_u32_host(out.ctypes.data, 10, 1, 256, 0) == bcf.BCF_ERROR_UNSUPPORTED
    assert L.bcf_worst_case_u32_host(out.ctypes.data, 10, 15, 100, 0) == bcf.BCF_ERROR_UNSUPPORTED


def test_merge_u32_query_and_validation():
    L = bcf.lib()
    tb = ctypes.c_size_t(0)
    assert L.bcf_merge_u32(None, 100, None, 100, None, None, None, None, None, ctypes.byref(tb), None, None) == 0
    need = tb.value
    assert 0 < need <= 1024 + 4 * 100
    tbp = ctypes.c_size_t(0)
    fake0 = ctypes.c_void_p(4096)
    assert L.bcf_merge_u32(None, 100, None, 100, fake0, fake0, None, fake0, None, ctypes.byref(tbp), None,
                           None) == 0 and 0 < tbp.value <= 512 + 2 * 768
    assert L.bcf_merge_u32(None, 1, None, 1, None, None, None, None, None, None, None,
                           None) == bcf.BCF_ERROR_INVALID_VALUE
    small = ctypes.c_size_t(need - 1)
    assert L.bcf_merge_u32(None, 100, None, 100, None, None, None, None, ctypes.c_void_p(256), ctypes.byref(small),
                           None, None) == bcf.BCF_ERROR_TEMP_TOO_SMALL
    tb = ctypes.c_size_t(need)
    tmp = ctypes.c_void_p(256)
    # na = nb = 0 is a no-op; null inputs / output with data are rejected before any launch
    assert L.bcf_merge_u32(None, 0, None, 0, None, None, None, None, tmp, ctypes.byref(tb), None, None) == 0
    fake = ctypes.c_void_p(4096)
    assert L.bcf_merge_u32(None, 5, fake, 5, None, None, fake, None, tmp, ctypes.byref(tb), None,
                           None) == bcf.BCF_ERROR_INVALID_VALUE
    assert L.bcf_merge_u32(fake, 5, fake, 5, None, None, None, None, tmp, ctypes.byref(tb), None,
                           None) == bcf.BCF_ERROR_INVALID_VALUE
    # values: all three or none
    assert L.bcf_merge_u32(fake, 5, fake, 5, fake, None, fake, fake, tmp, ctypes.byref(tb), None,
                           None) == bcf.BCF_ERROR_INVALID_VALUE
    assert L.bcf_merge_u32(None, 5, None, 5, None, None, None, None, None, ctypes.byref(tb),
                           bcf.make_params(15, 256, bcf.ALGO_BASELINE), None) == bcf.BCF_ERROR_UNSUPPORTED
    assert L.bcf_merge_u32(None, 5, None, 5, None, None, None, None, None, ctypes.byref(tb),
                           bcf.make_params(18, 256), None) == bcf.BCF_ERROR_UNSUPPORTED


@pytest.mark.parametrize("E,u,n,seed", [
    (15, 64, 15 * 2 ** 9, 1234), (17, 64, 17 * 2 ** 9, 5), (16, 64, 2 ** 13, 7), (12, 64, 12 * 2 ** 9, 9),
    (8, 128, 2 ** 13, 11), (15, 256, 100000, 3), (16, 256, 2 ** 16, 0xB2000000), (9, 128, 7777, 1),
    (13, 512, 1, 2), (7, 128, 0, 3), (15, 512, 15 * 2 ** 14, 4), (11, 256, 50001, 8),
    (31, 128, 31 * 2 ** 12, 6), (31, 128, 100001, 7), (19, 64, 19 * 2 ** 10, 12), (24, 128, 24 * 2 ** 11, 13),
    (32, 64, 2 ** 14 + 3, 14), (2, 32, 5000, 15), (31, 256, 31 * 2 ** 13 + 17, 16),
])
def test_host_worst_case_matches_oracle(E, u, n, seed):
    got = bcf.worst_case_host(n, E, u, seed)
    exp = wc.worst_case_input(n, E, u, seed)
    np.testing.assert_array_equal(got, exp)


def test_host_worst_case_is_permutation_at_bench_size():
    n = 1 << 22
    x = bcf.worst_case_host(n, 16, 256, 0xB2000001)
    assert np.array_equal(np.sort(x), np.arange(n, dtype=np.uint32))


def test_host_worst_case_matches_oracle_at_the_bench_configuration():
    """BASELINE configs[1]: 2^24 keys for the default (E, u) = (31, 128)."""
    n = 1 << 24
    np.testing.assert_array_equal(bcf.worst_case_host(n, 31, 128, 0xB2000001),
                                  wc.worst_case_input(n, 31, 128, 0xB2000001))


def test_host_batch_query_and_validation():
    """bcf_sort_u32_host_batch: CUB-style temp query (two device slots of
    input + output keys plus the sort's own temp) and synchronous argument
    errors, all without touching a GPU."""
    L = bcf.lib()
    for n in [0, 1000, 1 << 24]:
        tb = ctypes.c_size_t(0)
        assert L.bcf_sort_u32_host_batch(None, None, 3, n, None, ctypes.byref(tb), None, None) == 0
        _, sort_tb = _query(L.bcf_sort_u32, n)
        assert tb.value >= 16 * n + sort_tb
    tb = ctypes.c_size_t(0)
    assert L.bcf_sort_u32_host_batch(None, None, -1, 10, None, ctypes.byref(tb), None,
                                     None) == bcf.BCF_ERROR_INVALID_VALUE
    assert L.bcf_sort_u32_host_batch(None, None, 1, 10, None, None, None, None) == bcf.BCF_ERROR_INVALID_VALUE
    assert L.bcf_sort_u32_host_batch(None, None, 1, 10, None, ctypes.byref(tb), ctypes.byref(bcf.make_params(18, 256)),
                                     None) == bcf.BCF_ERROR_UNSUPPORTED
    # null host arrays with a real temp pointer: rejected before any copy
    assert L.bcf_sort_u32_host_batch(None, None, 0, 10, None, ctypes.byref(tb), None, None) == 0
    need = tb.value
    tb = ctypes.c_size_t(need)
    assert L.bcf_sort_u32_host_batch(None, None, 2, 10, ctypes.c_void_p(256), ctypes.byref(tb), None,
                                     None) == bcf.BCF_ERROR_INVALID_VALUE


def test_sort_plan():
    """Pass plan: keys-only CF (31, 128) sorts block tiles of 2u threads; every
    other configuration (pairs, baseline, other E/u) keeps u; passes =
    ceil(log2(n / block tile))."""
    assert bcf.sort_plan(1 << 24) == {"block_sort_tile": 7936, "merge_tile": 3968, "merge_passes": 12}
    assert bcf.sort_plan(7936)["merge_passes"] == 0
    assert bcf.sort_plan(7937)["merge_passes"] == 1
    assert bcf.sort_plan(1 << 24, bcf.make_params(31, 128, bcf.ALGO_BASELINE)) == \
        {"block_sort_tile": 3968, "merge_tile": 3968, "merge_passes": 13}
    assert bcf.sort_plan(1 << 26, pairs=True) == {"block_sort_tile": 11 * 256, "merge_tile": 11 * 256,
                                                  "merge_passes": 15}  # ceil(log2(2^26 / 2816))
    assert bcf.sort_plan(1 << 26, bcf.make_params(17, 256), pairs=True)["merge_passes"] == 14
    assert bcf.sort_plan(1 << 24, bcf.make_params(15, 256)) == {"block_sort_tile": 3840, "merge_tile": 3840,
                                                               "merge_passes": 13}


def test_set_op_query_and_validation():
    """bcf_set_op_u32: CUB-style temp query and synchronous argument errors
    (no GPU needed)."""
    L = bcf.lib()
    tb = ctypes.c_size_t(0)
    assert L.bcf_set_op_u32(0, None, 1000, None, 2000, None, None, None, None, ctypes.byref(tb), None, None) == 0
    assert tb.value >= 4 * 3000 * 2  # merged keys + tags at least
    assert L.bcf_set_op_u32(4, None, 10, None, 10, None, None, None, None, ctypes.byref(tb), None,
                            None) == bcf.BCF_ERROR_INVALID_VALUE
    assert L.bcf_set_op_u32(-1, None, 10, None, 10, None, None, None, None, ctypes.byref(tb), None,
                            None) == bcf.BCF_ERROR_INVALID_VALUE
    assert L.bcf_set_op_u32(0, None, 1 << 31, None, 10, None, None, None, None, ctypes.byref(tb), None,
                            None) == bcf.BCF_ERROR_UNSUPPORTED
    big = ctypes.c_size_t(1 << 40)
    fake = ctypes.c_void_p(256)
    # count pointer missing
    assert L.bcf_set_op_u32(1, fake, 10, fake, 10, fake, None, None, fake, ctypes.byref(big), None,
                            None) == bcf.BCF_ERROR_INVALID_VALUE
