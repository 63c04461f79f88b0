"""Pins for oracle/worstcase.py: Lemmas 5-7, |T| = w/d, the per-subproblem
A/B counts, the two panels of Figure 4, Theorem 8's closed form against the
DMM simulation of the Thrust serial merge, and the multi-level composition
(every regular level drives the simulated Thrust merge to Theorem 8)."""
from math import ceil, floor, gcd

import numpy as np
import pytest

from conftest import grid_to_cells
from oracle import dmm
from oracle import worstcase as wc

W_SET = [12, 16, 24, 30, 32]


@pytest.mark.parametrize("w", W_SET)
def test_lemmas_5_6_7(w):
    for E in range(2, w + 1):
        d = gcd(w, E)
        q, r = wc.euclid(w, E)
        assert w == q * E + r and 0 <= r < E
        S = wc.S_sequence(w, E)
        s = {i: si for (i, si, _, _, _, _) in S}
        x = {i: xi for (i, _, xi, _, _, _) in S}
        y = {i: yi for (i, _, _, yi, _, _) in S}
        Ed, rd = E // d, r // d
        assert len(set(s.values())) == len(s)                       # Lemma 5
        for i in s:
            assert Ed - s[i] == s[Ed - i]                            # Lemma 6
        for i in range(1, Ed - 1):                                   # Lemma 7
            exp = r if s[i] > Ed - rd else E + r
            assert x[i] + y[i + 1] == exp


@pytest.mark.parametrize("w", W_SET)
def test_T_length_and_counts(w):
    for E in range(2, w + 1):
        d = gcd(w, E)
        T = wc.T_sequence(w, E)
        assert len(T) == w // d
        assert all(a + b == E and a >= 0 and b >= 0 for a, b in T)
        # per subproblem ceil(E/2d) w elements of A and floor(E/2d) w of B
        # (reading c6)
        assert sum(a for a, _ in T) == ceil(E / (2 * d)) * w
        assert sum(b for _, b in T) == floor(E / (2 * d)) * w


def _thrust_owner_grid(w, E, tuples):
    """Thrust layout: A then B (not reversed); owner of every cell."""
    A, B = [], []
    for t, (a, b) in enumerate(tuples):
        A += [t] * a
        B += [t] * b
    return A + B


@pytest.mark.parametrize("name", ["fig4_w12_E5_worstcase.txt", "fig4_w12_E9_worstcase.txt"])
def test_fig4_panels(golden, name):
    p, rows, _ = golden(name)
    w, E = p["w"], p["E"]
    cells = _thrust_owner_grid(w, E, wc.warp_thread_tuples(w, E))
    assert cells == grid_to_cells(rows)


def _simulate_warp_serial_merge(w, E, tuples):
    d = gcd(w, E)
    labels = []
    for idx, (a, b) in enumerate(tuples):
        sub = idx // (w // d)
        labels += ([True] * b + [False] * a) if sub % 2 == 0 else ([False] * a + [True] * b)
    A = [o for o, l in enumerate(labels) if not l]
    B = [o for o, l in enumerate(labels) if l]
    smem = A + B
    streams, a, b = [], 0, 0
    for (ta, tb) in tuples:
        streams.append(dmm.serial_merge_addresses(smem, a, len(A) + b, ta, tb, E))
        a += ta
        b += tb
    return dmm.warp_instruction_conflicts(streams, w)


@pytest.mark.parametrize("E", list(range(2, 19)) + [20, 21, 32])
def test_theorem8_matches_simulated_serial_merge(E):
    """Theorem 8 (combined) = simulated extra wavefronts of the
    warp's serial merge + 1 (conflict-count convention, reading c14).  The
    paper's figures and formulas are for 1 < E <= w; E in {19, 22..31} need an
    interleaving the paper does not specify (reading c9) and are not claimed."""
    w = 32
    sim = _simulate_warp_serial_merge(w, E, wc.warp_thread_tuples(w, E))
    assert sim + 1 == wc.theorem8_warp(w, E)


def test_theorem8_case_formulas():
    # Case 1 (E <= w/2): E^2 / d per subproblem, E^2 per warp
    assert wc.theorem8_subproblem(32, 15) == 225
    assert wc.theorem8_warp(32, 12) == 144
    # Case 2: 1/2 (E^2 + 2Er + Ed - r^2 - rd); w = 32, E = 17: q = 1, r = 15
    assert wc.theorem8_warp(32, 17) == 0.5 * (289 + 2 * 17 * 15 + 17 - 225 - 15)
    # d = E => r = 0 and no element is misaligned
    assert wc.theorem8_subproblem(32, 32) == 32


# ---- multi-level composition -------------------------------------------------

def _thrust_level_conflicts(keys, R, E, u, w=32):
    """Simulate one merge level (runs of R -> 2R) of the Thrust mergesort on
    `keys` (runs of R already sorted); returns (merged keys, per-warp conflict
    list for regular groups).  Thread splits come from the stable-merge
    definition; block-sort levels use a group of 2R/E threads, global passes
    tiles of uE outputs."""
    n = len(keys)
    out = np.empty_like(keys)
    per_warp = []
    tile = u * E
    for g0 in range(0, n, 2 * R):
        A = keys[g0:min(n, g0 + R)]
        B = keys[min(n, g0 + R):min(n, g0 + 2 * R)]
        merged_lab = []
        i = j = 0
        while i < len(A) or j < len(B):
            if j < len(B) and (i >= len(A) or B[j] < A[i]):
                merged_lab.append(("B", j)); j += 1
            else:
                merged_lab.append(("A", i)); i += 1
        out[g0:g0 + len(merged_lab)] = [A[x] if l == "A" else B[x] for l, x in merged_lab]
        regular = (len(A) == R and len(B) == R and R % (w * E) == 0)
        if not regular:
            continue
        span = tile if 2 * R > tile else 2 * R      # merge tile (global) or whole group
        for t0 in range(0, 2 * R, span):
            lab = merged_lab[t0:t0 + span]
            a0 = sum(1 for l, _ in merged_lab[:t0] if l == "A")
            b0 = t0 - a0
            nA = sum(1 for l, _ in lab if l == "A")
            smem = list(A[a0:a0 + nA]) + list(B[b0:b0 + span - nA])
            for v0 in range(0, span, w * E):
                streams = []
                for t in range(v0 // E, v0 // E + w):
                    seg = lab[t * E:(t + 1) * E]
                    a = sum(1 for l, _ in lab[:t * E] if l == "A")
                    b = t * E - a
                    na = sum(1 for l, _ in seg if l == "A")
                    streams.append(dmm.serial_merge_addresses(smem, a, nA + b, na, E - na, E))
                per_warp.append(dmm.warp_instruction_conflicts(streams, w))
    return out, per_warp


@pytest.mark.parametrize("E,u,n", [(15, 64, 15 * 2 ** 9), (17, 64, 17 * 2 ** 9),
                                   (16, 64, 2 ** 13), (12, 64, 12 * 2 ** 9), (8, 128, 2 ** 13)])
def test_composition_hits_theorem8_at_every_regular_level(E, u, n):
    w = 32
    x = wc.worst_case_input(n, E, u, seed=1234)
    assert sorted(x.tolist()) == list(range(n))              # a permutation of ranks
    np.testing.assert_array_equal(x, wc.worst_case_input(n, E, u, seed=1234))  # deterministic
    # bottom-up simulation of the sort: runs of E first
    keys = x.astype(np.int64).copy()
    for s in range(0, n, E):
        keys[s:s + E] = np.sort(keys[s:s + E])
    thm = wc.theorem8_warp(w, E)
    regular_levels = 0
    for R in wc.merge_levels(n, E, u):
        keys, per_warp = _thrust_level_conflicts(keys, R, E, u, w)
        if per_warp:
            regular_levels += 1
            assert all(c + 1 == thm for c in per_warp), (R, set(per_warp))
    np.testing.assert_array_equal(keys, np.arange(n))
    assert regular_levels >= 3


def test_composition_ragged_sizes_are_permutations():
    for n in [0, 1, 14, 15, 16, 1000, 3841, 9999]:
        x = wc.worst_case_input(n, 15, 64, seed=9)
        assert sorted(x.tolist()) == list(range(n))
