"""Pins for oracle/addrmap.py and oracle/dmm.py: the paper's worked examples
(Figs. 2, 3, 7), the number-theoretic facts (Lemma 1, Lemma 2/Cor. 3) checked
by brute force, and Alg. 1 on random merges whose splits come from the plain
definition of a stable merge."""
from math import gcd

import numpy as np
import pytest

from conftest import grid_to_cells, splits_from_comments
from oracle import addrmap as am
from oracle import dmm


def splits_to_offsets(splits):
    """[(nA, nB)] -> [(a_i, b_i, nA, nB)] with a_i, b_i prefix sums."""
    out, a, b = [], 0, 0
    for na, nb in splits:
        out.append((a, b, na, nb))
        a += na
        b += nb
    return out, a, b


# ---- rho -------------------------------------------------------------------

@pytest.mark.parametrize("w", [6, 9, 12, 32])
def test_rho_is_bijection_and_inverse(w):
    for E in range(1, 2 * w + 1):
        T = 4 * w * E
        img = [am.rho(k, w, E) for k in range(T)]
        assert sorted(img) == list(range(T))
        assert all(am.rho_inv(am.rho(k, w, E), w, E) == k for k in range(T))
        if gcd(w, E) == 1:
            assert img == list(range(T))  # d = 1: rho is the identity


def _round_sets_conflict_free(w, E, mapping):
    """Brute force over every window start alpha and round j: the w logical
    indices that are = j (mod E) inside [alpha, alpha + wE) must land in w
    distinct banks (Lemma 1 for d = 1; Lemma 2 / Cor. 3 + §3.3 for d > 1)."""
    span = w * E
    # the layout repeats every d partitions = wE elements, so alpha in [0, wE)
    # covers every window; check 2 periods to include the wrap.
    phys = np.array([mapping(k) for k in range(4 * span)])
    k = np.arange(2 * span)[:, None] + np.arange(span)[None, :]      # windows
    key = (k % E) * w + (phys[k] % w)          # (round, bank) of every element
    key.sort(axis=1)
    return bool(np.all(np.diff(key, axis=1) != 0))


@pytest.mark.parametrize("w", [6, 9, 12, 32])
def test_lemma1_cor3_complete_residue_systems(w):
    for E in range(1, 2 * w + 1):
        ok_rho = _round_sets_conflict_free(w, E, lambda k: am.rho(k, w, E))
        assert ok_rho, (w, E)
        ok_id = _round_sets_conflict_free(w, E, lambda k: k)
        # without rho the round sets conflict exactly when w and E are not coprime
        assert ok_id == (gcd(w, E) == 1), (w, E)


# ---- Figures ----------------------------------------------------------------

def test_fig2_layout_and_one_read_per_round(golden):
    p, rows, comments = golden("fig2_w12_E5_reversed.txt")
    w, E = p["w"], p["E"]
    splits, NA, NB = splits_to_offsets(splits_from_comments(comments))
    cells = am.layout_owner_grid(splits, NA, NB, w, E, reverse_B=True)
    assert cells == grid_to_cells(rows)
    for j in range(E):
        addrs = []
        for t, (a, b, na, nb) in enumerate(splits):
            idx, _ = am.gather_indices(a, b, na, nb, NA, NB, w, E)[j]
            assert cells[idx] == t
            addrs.append(idx)
        assert dmm.conflicts(addrs, w) == 0
    # every thread reads each of its E cells exactly once over the E rounds
    for t, (a, b, na, nb) in enumerate(splits):
        got = sorted(i for i, _ in am.gather_indices(a, b, na, nb, NA, NB, w, E))
        assert got == sorted(k for k, o in enumerate(cells) if o == t)


def _max_reads_per_round(cells, E):
    """Reading A_i and B_i each in ascending round order (round = address mod
    E): the largest number of a thread's cells that fall in one round."""
    worst = 0
    for t in set(cells):
        rounds = [k % E for k, o in enumerate(cells) if o == t]
        worst = max(worst, max(rounds.count(r) for r in set(rounds)))
    return worst


def test_fig7_forward_B_needs_two_reads_per_round(golden):
    p, rows, comments = golden("fig7_w12_E5_forward.txt")
    w, E = p["w"], p["E"]
    splits, NA, NB = splits_to_offsets(splits_from_comments(comments))
    fwd = am.layout_owner_grid(splits, NA, NB, w, E, reverse_B=False)
    assert fwd == grid_to_cells(rows)
    assert _max_reads_per_round(fwd, E) == 2          # Fig. 7: stalls
    rev = am.layout_owner_grid(splits, NA, NB, w, E, reverse_B=True)
    assert _max_reads_per_round(rev, E) == 1          # §3.1: reversal fixes it


def _ownership_valid(logical, E):
    """A logical (pre-rho) ownership sequence is a valid 'A then reversed B'
    layout: thread ids non-decreasing over a prefix, non-increasing over the
    rest, every thread owning E cells."""
    n = len(logical)
    for cut in range(n + 1):
        A, B = logical[:cut], logical[cut:]
        if all(A[i] <= A[i + 1] for i in range(len(A) - 1)) and all(
            B[i] >= B[i + 1] for i in range(len(B) - 1)
        ):
            if all(logical.count(t) == E for t in set(logical)):
                return True
    return False


def test_fig3_rho_rotates_right(golden):
    p, rows, _ = golden("fig3_w9_E6_rho.txt")
    w, E = p["w"], p["E"]
    cells = grid_to_cells(rows)
    T = len(cells)
    assert am.partition_size(w, E) == 18           # caption's "16" is a typo (c4)
    logical = [cells[am.rho(k, w, E)] for k in range(T)]
    assert _ownership_valid(logical, E)
    # rotating LEFT instead does not give a valid A / reversed-B preimage
    P, d = am.partition_size(w, E), gcd(w, E)

    def rho_left(k):
        l, x = divmod(k, P)
        return l * P + (x - (l % d)) % P

    assert not _ownership_valid([cells[rho_left(k)] for k in range(T)], E)
    # every round of Alg. 1 on the recovered splits is conflict-free
    cut = next(c for c in range(T + 1)
               if all(logical[i] <= logical[i + 1] for i in range(c - 1))
               and all(logical[i] >= logical[i + 1] for i in range(c, T - 1)))
    A, Brev = logical[:cut], logical[cut:]
    B = Brev[::-1]
    splits, NA, NB = splits_to_offsets([(A.count(t), B.count(t)) for t in range(w)])
    for j in range(E):
        addrs = [am.gather_indices(a, b, na, nb, NA, NB, w, E)[j][0]
                 for (a, b, na, nb) in splits]
        assert dmm.conflicts(addrs, w) == 0


# ---- Alg. 1 on random merges (splits from the plain definition) -------------

def stable_merge_labels(A, B):
    """Plain definition: stable merge of sorted A and B (ties to A); returns
    the list of 'A'/'B' labels of the outputs."""
    i = j = 0
    lab = []
    while i < len(A) or j < len(B):
        if j < len(B) and (i >= len(A) or B[j] < A[i]):
            lab.append("B")
            j += 1
        else:
            lab.append("A")
            i += 1
    return lab


def splits_by_definition(A, B, E, nthreads):
    lab = stable_merge_labels(A, B)
    out = []
    for t in range(nthreads):
        seg = lab[t * E:(t + 1) * E]
        a = lab[:t * E].count("A")
        b = lab[:t * E].count("B")
        out.append((a, b, seg.count("A"), seg.count("B")))
    return out


@pytest.mark.parametrize("E", list(range(5, 18)))
@pytest.mark.parametrize("u", [64, 128])
def test_alg1_gather_conflict_free_and_complete(E, u):
    w = 32
    rng = np.random.default_rng(E * 1000 + u)
    for trial in range(6):
        T = u * E
        vals = rng.integers(0, 4 if trial % 2 else 1 << 30, size=T)
        NA = int(rng.integers(0, T + 1)) if trial > 1 else T // 2
        A = sorted(vals[:NA].tolist())
        B = sorted(vals[NA:].tolist())
        NB = T - NA
        splits = splits_by_definition(A, B, E, u)
        smem = [None] * T
        for x in range(NA):
            smem[am.rho(x, w, E)] = ("A", x)
        for y in range(NB):
            smem[am.rho(am.pi_B(y, NA, NB), w, E)] = ("B", y)
        for v in range(u // w):
            for j in range(E):
                addrs = []
                for t in range(v * w, (v + 1) * w):
                    idx, elem = am.gather_indices(*splits[t], NA, NB, w, E)[j]
                    assert smem[idx] == elem
                    addrs.append(idx)
                assert dmm.conflicts(addrs, w) == 0, (E, u, v, j)
        # each thread gathers exactly A_i and B_i
        for t, (a, b, na, nb) in enumerate(splits):
            got = {e for _, e in am.gather_indices(a, b, na, nb, NA, NB, w, E)}
            assert got == {("A", x) for x in range(a, a + na)} | {("B", y) for y in range(b, b + nb)}


def test_dmm_wavefront_model():
    assert dmm.wavefronts(list(range(32))) == 1
    assert dmm.wavefronts([0] * 32) == 1                      # broadcast
    assert dmm.wavefronts([2 * i for i in range(32)]) == 2    # stride 2: 2-way
    assert dmm.wavefronts([32 * i for i in range(32)]) == 32  # same bank
    assert dmm.wavefronts([5 * i for i in range(12)], w=12) == 1   # Fig. 1 left
    assert dmm.wavefronts([6 * i for i in range(12)], w=12) == 6   # Fig. 1 right
    assert dmm.wavefronts([None] * 32) == 0
