"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element, bit-exact (tolerance 0: north_star).  Sizes span several
tiles, ragged tails, single-tile and edge cases; every instantiated (E, u)
and both algorithms; f32 special values; stable pairs; in-place and
unaligned buffers; the merge_runs / split_counts phases; the worst-case
generator; and the full BASELINE sizes in the bench launch configuration."""
import numpy as np
import pytest

import oracle
import synthetic_inputs as si

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")


def to_dev(a: np.ndarray):
    return torch.from_numpy(a.view(np.int32).copy()).to(DEV)


def to_host(t) -> np.ndarray:
    return t.cpu().numpy().view(np.uint32)


def gpu_sort_u32(x: np.ndarray, params=None):
    out = bcf.sort(to_dev(x), params=params)
    torch.cuda.synchronize()
    return to_host(out)


SIZES = [1, 2, 15, 16, 17, 255, 4095, 4096, 4097, 8191, 8192, 12289, 3840 * 3 + 7, 65536, 100003, 262144 + 77]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("kind", ["uniform", "dup"])
def test_default_u32_parity(n, kind):
    seed = si.config_seed(0) + n
    x = si.uniform_u32(n, seed) if kind == "uniform" else si.dup_u32(n, seed, mask=0x3)
    np.testing.assert_array_equal(gpu_sort_u32(x), oracle.sort_u32(x))


@pytest.mark.parametrize("E", list(range(7, 18)) + [31])
@pytest.mark.parametrize("u", [128, 256, 512])
@pytest.mark.parametrize("algo", [bcf.ALGO_CONFLICT_FREE, bcf.ALGO_BASELINE])
def test_all_instantiations_u32(E, u, algo):
    T = E * u
    for n in [T - 1, 5 * T + 3, 9 * T]:
        x = si.uniform_u32(n, si.config_seed(3) + E * 1000 + u + n)
        if n % 2:
            x &= np.uint32(0xF)  # duplicates
        got = gpu_sort_u32(x, bcf.make_params(E, u, algo))
        np.testing.assert_array_equal(got, oracle.sort_u32(x), err_msg=f"E={E} u={u} algo={algo} n={n}")


@pytest.mark.parametrize("kind", ["sorted", "reversed", "equal", "organ", "worst"])
def test_structured_inputs(kind):
    n = 200000
    if kind == "sorted":
        x = np.arange(n, dtype=np.uint32)
    elif kind == "reversed":
        x = np.arange(n, dtype=np.uint32)[::-1].copy()
    elif kind == "equal":
        x = np.full(n, 0xFFFFFFFF, np.uint32)
    elif kind == "organ":
        x = np.concatenate([np.arange(n // 2), np.arange(n - n // 2)[::-1]]).astype(np.uint32)
    else:
        p = bcf.default_params()
        x = bcf.worst_case_host(n, p.items_per_thread, p.block_threads, 1)
    np.testing.assert_array_equal(gpu_sort_u32(x), oracle.sort_u32(x))


def _skewed(kind: str, n: int, seed: int) -> np.ndarray:
    """Inputs whose merge paths leave the predicted windows of the persistent
    merge pass (bcf_merge_win.cuh): the A share of consecutive subtiles jumps
    between 0 and 1, drifts, or differs between the two runs of a group."""
    h = si.uniform_u32(n, seed)
    i = np.arange(n, dtype=np.uint64)
    if kind == "sawtooth":          # sorted segments of random length
        seg = np.cumsum(1 + (si.uniform_u32(n // 64 + 2, seed + 1) % 20000)).astype(np.int64)
        start = np.zeros(n, np.int64)
        idx = np.searchsorted(seg, np.arange(n), side="right")
        start[:] = np.concatenate([[0], seg])[idx]
        return (np.arange(n) - start).astype(np.uint32) * np.uint32(977)
    if kind == "bands":             # chunks drawn from disjoint key bands
        band = (i // 3000) % 7
        return ((band.astype(np.uint32) << np.uint32(28)) | (h >> np.uint32(4))).astype(np.uint32)
    if kind == "scaled":            # uniform, each 1000-chunk scaled differently
        f = si.uniform_u32(n // 1000 + 1, seed + 2)[i // 1000] >> np.uint32(24)
        return ((h >> np.uint32(8)) * (f + np.uint32(1))).astype(np.uint32)
    if kind == "nearly_sorted":     # sorted with 1 % random swaps
        x = np.arange(n, dtype=np.uint32)
        k = n // 100
        a = si.uniform_u32(k, seed + 3) % n
        b = si.uniform_u32(k, seed + 4) % n
        for p, q in zip(a, b):
            x[p], x[q] = x[q], x[p]
        return x
    raise ValueError(kind)


@pytest.mark.parametrize("kind", ["sawtooth", "bands", "scaled", "nearly_sorted"])
@pytest.mark.parametrize("E,u", [(31, 128), (15, 256), (9, 128), (31, 256), (17, 512)])
def test_skewed_window_exhaustion(kind, E, u):
    # the persistent merge pass ends a subtile early when the merge path
    # leaves a window; parity must hold for every such subtile
    n = 300000 + 13
    x = _skewed(kind, n, si.config_seed(6) + E * 7 + u)
    got = gpu_sort_u32(x, bcf.make_params(E, u, bcf.ALGO_CONFLICT_FREE))
    np.testing.assert_array_equal(got, oracle.sort_u32(x), err_msg=f"{kind} E={E} u={u}")


def test_extreme_keys_and_pads():
    # real UINT32_MAX keys in a ragged last tile must not be confused with pads
    for n in [4097, 100001]:
        x = si.uniform_u32(n, 77 + n)
        x[::3] = 0xFFFFFFFF
        x[1::7] = 0
        np.testing.assert_array_equal(gpu_sort_u32(x), oracle.sort_u32(x))


@pytest.mark.parametrize("n", [1, 1000, 4096, 65537, 300000])
def test_f32_total_order(n):
    bits = si.special_f32_bits(n, si.config_seed(2) + n)
    t = to_dev(bits).view(torch.float32)
    out = bcf.sort(t)
    torch.cuda.synchronize()
    got = out.view(torch.int32).cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(got, oracle.sort_f32_bits(bits))


def test_f32_uniform():
    n = 1 << 20
    x = si.uniform_f32(n, si.config_seed(2))
    out = bcf.sort(torch.from_numpy(x).to(DEV))
    got = out.cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(got, oracle.sort_f32_bits(x.view(np.uint32)))


@pytest.mark.parametrize("E,u", [(16, 256), (15, 256), (17, 128), (8, 512), (12, 256), (7, 128), (16, 512), (31, 128)])
@pytest.mark.parametrize("n", [1, 17, 4097, 100000])
def test_pairs_stable(E, u, n):
    k = si.dup_u32(n, si.config_seed(4) + n, mask=0xF)
    v = si.iota_u32(n)
    ko, vo = bcf.sort_pairs(to_dev(k), to_dev(v), params=bcf.make_params(E, u))
    ek, ev = oracle.sort_pairs_u32(k, v)
    np.testing.assert_array_equal(to_host(ko), ek)
    np.testing.assert_array_equal(to_host(vo), ev)


def test_in_place_and_unaligned():
    for n in [5000, 4096 * 4 + 1]:
        x = si.uniform_u32(n, 99 + n)
        t = to_dev(x)
        bcf.sort(t, out=t)  # in place
        np.testing.assert_array_equal(to_host(t), oracle.sort_u32(x))
        big = torch.zeros(n + 3, dtype=torch.int32, device=DEV)
        src = big[1:n + 1]
        src.copy_(to_dev(x))
        dst_big = torch.zeros(n + 5, dtype=torch.int32, device=DEV)
        dst = dst_big[3:n + 3]
        bcf.sort(src, out=dst)
        np.testing.assert_array_equal(to_host(dst), oracle.sort_u32(x))
        assert int(dst_big[0]) == 0 and int(dst_big[n + 3]) == 0  # no writes outside


@pytest.mark.parametrize("n", [3000, 200001, 1 << 20])
def test_pairs_unaligned_mismatched_phases(n):
    """Key and value buffers at different 16-byte phases (inputs and outputs):
    the persistent kernels' bulk stores assume one phase, so such a final pass
    must take the plain kernel; sort_pairs, merge_runs and merge stay exact."""
    k = si.dup_u32(n, si.config_seed(4) + n)
    v = si.iota_u32(n)
    ek, ev = oracle.sort_pairs_u32(k, v)

    def view(x, off):
        big = torch.zeros(x.size + 4, dtype=torch.int32, device=DEV)
        t = big[off:off + x.size]
        t.copy_(to_dev(x))
        return t

    kin, vin = view(k, 1), view(v, 2)
    kout, vout = view(np.zeros(n, np.uint32), 3), view(np.zeros(n, np.uint32), 0)
    bcf.sort_pairs(kin, vin, kout, vout)
    np.testing.assert_array_equal(to_host(kout), ek)
    np.testing.assert_array_equal(to_host(vout), ev)
    # two sorted halves -> merge (pairs), outputs at different phases
    h = n // 2
    ak, av = oracle.sort_pairs_u32(k[:h], v[:h])
    bk, bv = oracle.sort_pairs_u32(k[h:], v[h:])
    mk, mv = oracle.sort_pairs_u32(np.concatenate([ak, bk]), np.concatenate([av, bv]))
    for aoff, ooff in ((0, 0), (1, 2), (0, 3)):
        ko, vo = view(np.zeros(n, np.uint32), ooff), view(np.zeros(n, np.uint32), 0)
        bcf.merge(view(ak, aoff), view(bk, 0), view(av, 0), view(bv, 1), out=ko, out_values=vo)
        np.testing.assert_array_equal(to_host(ko), mk)
        np.testing.assert_array_equal(to_host(vo), mv)


def test_cuda_graph_capture_sort_and_merge():
    """The sort and bcf_merge_u32 are kernel launches only: captured once into
    a CUDA graph, each replay re-sorts / re-merges the current buffer contents."""
    n = (1 << 20) + 17
    x = to_dev(si.uniform_u32(n, 11))
    out = torch.empty_like(x)
    temp = bcf.temp_buffer(n, device=DEV)
    a0 = np.sort(si.uniform_u32(70001, 12))
    b0 = np.sort(si.uniform_u32(50003, 13))
    a, b = to_dev(a0), to_dev(b0)
    mo = torch.empty(a.numel() + b.numel(), dtype=torch.int32, device=DEV)
    mtemp = bcf.merge_temp(a.numel(), b.numel(), device=DEV)
    bcf.sort(x, out=out, temp=temp)  # warm-up outside the capture (attribute caches)
    bcf.merge(a, b, out=mo, temp=mtemp)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        bcf.sort(x, out=out, temp=temp)
        bcf.merge(a, b, out=mo, temp=mtemp)
    for seed in (21, 22):
        xs = si.uniform_u32(n, seed)
        x.copy_(to_dev(xs))
        a1 = np.sort(si.uniform_u32(70001, seed + 100))
        b1 = np.sort(si.uniform_u32(50003, seed + 200))
        a.copy_(to_dev(a1))
        b.copy_(to_dev(b1))
        g.replay()
        torch.cuda.synchronize()
        np.testing.assert_array_equal(to_host(out), oracle.sort_u32(xs))
        np.testing.assert_array_equal(to_host(mo), oracle.sort_u32(np.concatenate([a1, b1])))


def test_input_untouched():
    x = si.uniform_u32(50000, 5)
    t = to_dev(x)
    bcf.sort(t)
    np.testing.assert_array_equal(to_host(t), x)


def test_worst_case_device_matches_oracle():
    for (E, u, n) in [(16, 256, 1 << 16), (15, 256, 15 * 2 ** 12), (17, 256, 100000), (31, 128, 1 << 22),
                      (31, 128, 31 * 2 ** 15 + 7), (24, 64, 24 * 2 ** 12), (2, 32, 999)]:
        t = bcf.worst_case(n, E, u, seed=42, device=DEV)
        from oracle import worstcase as wc
        np.testing.assert_array_equal(to_host(t), wc.worst_case_input(n, E, u, 42))


def test_split_counts():
    x = np.sort(si.dup_u32(100000, 3, mask=0xFF))
    piv = np.array([0, 1, 5, 100, 255, 256, 0xFFFFFFFF], dtype=np.uint32)
    lt, le = bcf.split_counts(to_dev(x), to_dev(piv))
    np.testing.assert_array_equal(lt.cpu().numpy(), np.searchsorted(x, piv, side="left"))
    np.testing.assert_array_equal(le.cpu().numpy(), np.searchsorted(x, piv, side="right"))


@pytest.mark.parametrize("sizes", [[5], [3, 4], [0, 10, 0, 7], [4096, 4097, 1, 9000, 12345],
                                   [1000] * 8, [70000, 3, 70000]])
def test_merge_runs_stable(sizes):
    rng = np.random.default_rng(len(sizes) + sum(sizes))
    runs = [np.sort(rng.integers(0, 50, size=s).astype(np.uint32), kind="stable") for s in sizes]
    keys = np.concatenate(runs) if runs else np.zeros(0, np.uint32)
    vals = np.arange(keys.size, dtype=np.uint32)
    offs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.uint64)
    ko, vo = bcf.merge_runs(to_dev(keys), offs, values=to_dev(vals))
    ek, ev = oracle.sort_pairs_u32(keys, vals)  # stable sort of the concatenation
    np.testing.assert_array_equal(to_host(ko), ek)
    np.testing.assert_array_equal(to_host(vo), ev)
    k_only = bcf.merge_runs(to_dev(keys), offs)
    np.testing.assert_array_equal(to_host(k_only), ek)


@pytest.mark.parametrize("sizes", [[300001, 299999, 12345, 500000, 7, 250000, 0, 333333],
                                   [1 << 20] * 4, [123457] * 5, [2, 3, 5, 7, 11, 13, 17]])
@pytest.mark.parametrize("keyspace", [50, 1 << 32])
@pytest.mark.parametrize("params", [None, "15x256"])
def test_merge_runs_large(sizes, keyspace, params):
    """bcf_merge_runs_u32 at sizes spanning many tiles and CTAs: pass 1 on the
    plain kernel (ascending runs), later passes on the persistent TMA/window
    kernels over CF run directions; keys only and pairs."""
    prm = bcf.make_params(15, 256) if params else None
    rng = np.random.default_rng(sum(sizes) + keyspace % 97)
    runs = [np.sort(rng.integers(0, keyspace, size=s, dtype=np.uint64).astype(np.uint32), kind="stable")
            for s in sizes]
    keys = np.concatenate(runs)
    vals = np.arange(keys.size, dtype=np.uint32)
    offs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.uint64)
    ek, ev = oracle.sort_pairs_u32(keys, vals)
    ko = bcf.merge_runs(to_dev(keys), offs, params=prm)
    np.testing.assert_array_equal(to_host(ko), ek)
    ko, vo = bcf.merge_runs(to_dev(keys), offs, values=to_dev(vals), params=prm)
    np.testing.assert_array_equal(to_host(ko), ek)
    np.testing.assert_array_equal(to_host(vo), ev)


@pytest.mark.parametrize("nruns", [54, 62, 64])
def test_merge_runs_many_runs_with_empty_a_runs(nruns):
    """with nearly empty A (even) runs, pass 1 places every reversed
    B run at up to 3 phase words + an 8-word gap; the temp layout must hold
    ~11 extra words per B run (62 runs, odd runs of 49..79 keys)."""
    rng = np.random.default_rng(nruns)
    sizes = [0 if r % 2 == 0 else 49 + (r * 7) % 31 for r in range(nruns)]
    runs = [np.sort(rng.integers(0, 1 << 32, size=s, dtype=np.uint64).astype(np.uint32)) for s in sizes]
    keys = np.concatenate(runs)
    vals = np.arange(keys.size, dtype=np.uint32)
    offs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.uint64)
    ek, ev = oracle.sort_pairs_u32(keys, vals)
    np.testing.assert_array_equal(to_host(bcf.merge_runs(to_dev(keys), offs)), ek)
    ko, vo = bcf.merge_runs(to_dev(keys), offs, values=to_dev(vals))
    np.testing.assert_array_equal(to_host(ko), ek)
    np.testing.assert_array_equal(to_host(vo), ev)


def test_wrappers_reject_bad_buffers():
    """The Python binding checks sizes and devices before any launch."""
    x = to_dev(si.uniform_u32(1000, 5))
    with pytest.raises(bcf.BcfError):
        bcf.sort(x, out=torch.empty(999, dtype=torch.int32, device=DEV))
    with pytest.raises(bcf.BcfError):
        bcf.sort_pairs(x, x.clone(), keys_out=torch.empty(10, dtype=torch.int32, device=DEV))
    with pytest.raises(bcf.BcfError):
        bcf.merge_runs(x, np.array([0, 500, 1001], dtype=np.uint64))
    with pytest.raises(bcf.BcfError):
        bcf.merge_runs(x, np.array([0, 500, 1000], dtype=np.uint64), values=x[:999].clone())
    with pytest.raises(bcf.BcfError):
        bcf.merge(x[:500], x[500:], a_values=x[:499].clone(), b_values=x[500:].clone())
    with pytest.raises(bcf.BcfError):
        bcf.sort_pairs(x, torch.zeros(1000, dtype=torch.int32))  # values on the CPU


MERGE_SIZES = [(0, 0), (0, 5), (7, 0), (1, 1), (3968 * 3 + 17, 5000), (100000, 1), (1, 100000),
               (70001, 70003), (4352, 4352), (1 << 20, (1 << 20) - 3)]


@pytest.mark.parametrize("na,nb", MERGE_SIZES)
@pytest.mark.parametrize("dist", ["dups", "uniform", "disjoint"])
def test_merge_two_arrays(na, nb, dist):
    """bcf_merge_u32 == stable sort of A ++ B (ties: A first), keys and pairs,
    default and pairs parameters; A and B in separate allocations."""
    rng = np.random.default_rng(na * 7 + nb + len(dist))
    if dist == "dups":
        a = rng.integers(0, 50, size=na).astype(np.uint32)
        b = rng.integers(0, 50, size=nb).astype(np.uint32)
    elif dist == "uniform":
        a = si.uniform_u32(na, si.config_seed(0))
        b = si.uniform_u32(nb, si.config_seed(0), lo=na)
    else:  # every B key below every A key: the merge path runs along one edge
        a = rng.integers(1 << 31, 1 << 32, size=na, dtype=np.uint64).astype(np.uint32)
        b = rng.integers(0, 1 << 31, size=nb, dtype=np.uint64).astype(np.uint32)
    a.sort(kind="stable")
    b.sort(kind="stable")
    cat = np.concatenate([a, b])
    idx = np.arange(na + nb, dtype=np.uint32)
    ek, ev = oracle.sort_pairs_u32(cat, idx)
    # keys only: window kernel (odd E, aligned A; B reversed into temp) and
    # the plain kernel (even E: rho != identity)
    for params in (None, bcf.make_params(15, 256), bcf.make_params(16, 128), bcf.make_params(31, 512)):
        ko = bcf.merge(to_dev(a), to_dev(b), params=params)
        np.testing.assert_array_equal(to_host(ko), ek)
    for params in (None, bcf.make_params(15, 256)):
        ko, vo = bcf.merge(to_dev(a), to_dev(b), to_dev(idx[:na]), to_dev(idx[na:]), params=params)
        np.testing.assert_array_equal(to_host(ko), ek)
        np.testing.assert_array_equal(to_host(vo), ev)


def test_merge_unaligned_views():
    rng = np.random.default_rng(3)
    a = np.sort(rng.integers(0, 1000, size=20001).astype(np.uint32))
    b = np.sort(rng.integers(0, 1000, size=30003).astype(np.uint32))
    da = to_dev(np.concatenate([np.array([7], np.uint32), a]))[1:]
    db = to_dev(np.concatenate([np.array([1, 2, 3], np.uint32), b]))[3:]
    assert da.numel() == a.size and db.numel() == b.size
    ek, _ = oracle.sort_pairs_u32(np.concatenate([a, b]), np.arange(a.size + b.size, dtype=np.uint32))
    np.testing.assert_array_equal(to_host(bcf.merge(da, db)), ek)


# ---- full BASELINE sizes, bench launch configuration ------------------------

def test_full_2p24_random_and_worst():
    n = 1 << 24
    p = bcf.default_params()
    x = si.uniform_u32(n, si.config_seed(1))
    np.testing.assert_array_equal(gpu_sort_u32(x), oracle.sort_u32(x))
    w = bcf.worst_case(n, p.items_per_thread, p.block_threads, si.config_seed(1), device=DEV)
    out = bcf.sort(w)
    np.testing.assert_array_equal(to_host(out), np.arange(n, dtype=np.uint32))


def test_full_2p26_pairs():
    n = 1 << 26
    k = si.dup_u32(n, si.config_seed(5), mask=0xFFFF)
    v = si.iota_u32(n)
    ko, vo = bcf.sort_pairs(to_dev(k), to_dev(v))
    ek, ev = oracle.sort_pairs_u32(k, v)
    np.testing.assert_array_equal(to_host(ko), ek)
    np.testing.assert_array_equal(to_host(vo), ev)


def test_full_2p28_f32_against_oracle():
    """BASELINE configs[2]: 2^28 f32 in the bench configuration, compared with
    the oracle (totalOrder mergesort, 1 core, ~40 s) element by element."""
    n = 1 << 28
    x = si.uniform_f32(n, si.config_seed(6))
    out = bcf.sort(torch.from_numpy(x).to(DEV))
    torch.cuda.synchronize()
    got = out.cpu().numpy().view(np.uint32)
    del out
    torch.cuda.empty_cache()
    np.testing.assert_array_equal(got, oracle.sort_f32_bits(x.view(np.uint32)))


def _chunked_device_u32(n, seed, chunk=1 << 27):
    t = torch.empty(n, dtype=torch.int32, device=DEV)
    for lo in range(0, n, chunk):
        hi = min(n, lo + chunk)
        t[lo:hi] = si.uniform_u32_torch(hi - lo, seed, DEV, lo=lo)
    return t


def _check_big_sort_against_oracle(x: np.ndarray, got: np.ndarray, nranges=6, width=1 << 21):
    """Exact oracle checks for a sort too large to replay whole on one core:
    (1) the output is non-decreasing and has the input's multiset of keys
    (per-16-bit-bucket counts); (2) for several key ranges [lo, hi) the output
    slice at positions [#(x < lo), #(x < hi)) equals the oracle's sort of the
    input keys in [lo, hi) -- element by element, including the slices at the
    very start and end of the output (the 64-bit tile offsets past 2^31)."""
    n = x.size
    step = 1 << 26
    for lo in range(0, n - 1, step):
        hi = min(n, lo + step + 1)
        assert np.all(got[lo + 1:hi] >= got[lo:hi - 1]), f"not sorted near {lo}"
    hx = np.zeros(1 << 16, np.int64)
    hg = np.zeros(1 << 16, np.int64)
    for lo in range(0, n, step):
        hx += np.bincount(x[lo:lo + step] >> 16, minlength=1 << 16)
        hg += np.bincount(got[lo:lo + step] >> 16, minlength=1 << 16)
    np.testing.assert_array_equal(hx, hg)
    kmax = int(got[-1])
    bounds = [0] + [int(v) for v in np.linspace(0, kmax, nranges)[1:-1]] + [max(0, kmax - width * 4)]
    for klo in bounds:
        khi = min(klo + width * 4, 1 << 32)
        sel = np.concatenate([x[lo:lo + step][(x[lo:lo + step] >= klo) & (x[lo:lo + step] < khi)]
                              for lo in range(0, n, step)])
        before = int(sum(np.count_nonzero(x[lo:lo + step] < klo) for lo in range(0, n, step)))
        exp = oracle.sort_u32(sel)
        np.testing.assert_array_equal(got[before:before + exp.size], exp, err_msg=f"key range [{klo}, {khi})")


def test_sort_past_2p31_keys():
    """n = 2^31 + 12345 (bcf.h promises n up to 2^32): the 64-bit tile offsets
    and per-pass group arithmetic past 2^31, uniform random keys and the
    Section-4 worst case (a permutation of 0..n-1, whose sorted order is
    0..n-1), checked against the oracle as in _check_big_sort_against_oracle."""
    n = (1 << 31) + 12345
    t = _chunked_device_u32(n, si.config_seed(7))
    out = bcf.sort(t)
    torch.cuda.synchronize()
    x = t.cpu().numpy().view(np.uint32)
    del t
    got = out.cpu().numpy().view(np.uint32)
    del out
    torch.cuda.empty_cache()
    _check_big_sort_against_oracle(x, got)
    del x, got
    w = bcf.worst_case(n, 31, 128, seed=si.config_seed(7))
    out = bcf.sort(w)
    torch.cuda.synchronize()
    del w
    ok = torch.equal(out, torch.arange(n, dtype=torch.int64, device=DEV).to(torch.int32))
    got_head = out[:1 << 20].cpu().numpy().view(np.uint32)
    del out
    torch.cuda.empty_cache()
    assert ok
    np.testing.assert_array_equal(got_head, np.arange(1 << 20, dtype=np.uint32))


@pytest.mark.parametrize("nbatch,n", [(1, 1), (3, 4097), (5, 100003), (4, 1 << 20)])
def test_host_batch_parity(nbatch, n):
    """bcf_sort_u32_host_batch: H2D / sort / D2H pipelined over host arrays
    (pinned and one pageable), every output against the oracle."""
    xs = []
    for i in range(nbatch):
        seed = si.config_seed(6) + 31 * i + n
        x = si.uniform_u32(n, seed) if i % 2 == 0 else bcf.worst_case_host(n, 31, 128, seed)
        xs.append(x)
    h_in = [torch.from_numpy(x.view(np.int32).copy()) for x in xs]
    h_in = [t.pin_memory() if i != 1 else t for i, t in enumerate(h_in)]
    h_out = [torch.empty(n, dtype=torch.int32).pin_memory() for _ in range(nbatch)]
    bcf.sort_host_batch(h_in, h_out, device=DEV)
    torch.cuda.synchronize()
    for i, x in enumerate(xs):
        np.testing.assert_array_equal(h_out[i].numpy().view(np.uint32), oracle.sort_u32(x), err_msg=f"batch {i}")
    # in place (h_out[i] is h_in[i])
    bcf.sort_host_batch(h_in, h_in, device=DEV)
    torch.cuda.synchronize()
    for i, x in enumerate(xs):
        np.testing.assert_array_equal(h_in[i].numpy().view(np.uint32), oracle.sort_u32(x), err_msg=f"in place {i}")


BS2_SIZES = [1, 7936, 7937, 15871, 15872, 15873, 15872 * 3 + 5, 100003, 1 << 20]


@pytest.mark.parametrize("n", BS2_SIZES)
@pytest.mark.parametrize("kind", ["uniform", "dup", "worst"])
def test_two_tile_block_sort(n, kind, monkeypatch):
    """The opt-in two-tile block sort (BCF_BS2=1): runs of 2 x 7936
    keys (both tiles sorted, then one more CF level in shared memory), one
    merge pass fewer; the plan reports it and the result is the oracle's."""
    monkeypatch.setenv("BCF_BS2", "1")
    plan = bcf.sort_plan(n)
    assert plan["block_sort_tile"] == 2 * 7936
    seed = si.config_seed(0) + n
    if kind == "worst":
        x = to_host(bcf.worst_case(n, 31, 128, seed=seed, device=DEV))
    else:
        x = si.uniform_u32(n, seed) if kind == "uniform" else si.dup_u32(n, seed, mask=0x3)
    np.testing.assert_array_equal(gpu_sort_u32(x), oracle.sort_u32(x))
    f = si.special_f32_bits(n, seed)
    fo = bcf.sort(torch.from_numpy(f.view(np.float32).copy()).to(DEV))
    np.testing.assert_array_equal(to_host(fo), oracle.sort_f32_bits(f))


def test_even_e_window_kernel_opt_in():
    """The persistent window kernel for even E (cp.async staging in rho's
    physical order; opt-in BCF_EVEN_WIN=1, read when the launch table is
    built): a fresh process sorts keys and stable pairs at every even E
    against the oracle."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = r'''
import sys
sys.path.insert(0, %r)
import numpy as np, torch
import oracle, synthetic_inputs as si, paper_conf_spaa_berneys25_b200 as bcf
dev = torch.device("cuda:0")
n = 90001
x = si.dup_u32(n, 11, mask=0xFFF)
v = si.iota_u32(n)
for E in (8, 10, 12, 14, 16):
    for u in (128, 256):
        p = bcf.make_params(E, u)
        out = bcf.sort(torch.from_numpy(x.view(np.int32).copy()).to(dev), params=p)
        assert np.array_equal(out.cpu().numpy().view(np.uint32), oracle.sort_u32(x)), (E, u)
        ko, vo = bcf.sort_pairs(torch.from_numpy(x.view(np.int32).copy()).to(dev),
                                torch.from_numpy(v.view(np.int32).copy()).to(dev), params=p)
        ek, ev = oracle.sort_pairs_u32(x, v)
        assert np.array_equal(ko.cpu().numpy().view(np.uint32), ek), (E, u, "pairs keys")
        assert np.array_equal(vo.cpu().numpy().view(np.uint32), ev), (E, u, "pairs values")
print("even-window ok")
''' % root
    env = dict(os.environ, BCF_EVEN_WIN="1")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "even-window ok" in r.stdout, r.stdout + r.stderr


def test_cuda_graph_capture_merge_runs():
    """bcf_merge_runs_u32 (the distributed sort's final merge) writes its
    per-pass descriptor tables with small kernels, so it can be captured into
    a CUDA graph; each replay re-merges the current run contents."""
    sizes = [30001, 29999, 12345, 50000, 7, 25000]
    offs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.uint64)
    def runs_for(seed):
        return np.concatenate([np.sort(si.uniform_u32(m, seed + i)) for i, m in enumerate(sizes)])
    r0 = runs_for(31)
    runs = to_dev(r0)
    out0 = bcf.merge_runs(runs, offs)  # warm-up outside the capture (attribute caches)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(to_host(out0), oracle.sort_u32(r0))
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        out = bcf.merge_runs(runs, offs)
    for seed in (41, 42):
        rs = runs_for(seed)
        runs.copy_(to_dev(rs))
        g.replay()
        torch.cuda.synchronize()
        np.testing.assert_array_equal(to_host(out), oracle.sort_u32(rs))
