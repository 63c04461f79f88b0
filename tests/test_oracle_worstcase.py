"""Pins for oracle/worstcase.py: Lemmas 5-7, |T| = w/d, the per-subproblem
A/B counts, the two panels of Figure 4, Theorem 8's closed form against the
DMM simulation of the Thrust serial merge (the lockstep scan the proof counts
is exactly Theorem 8; the total is >= Theorem 8 and a local maximum over each
thread's interleaving), and the multi-level composition (every regular level
drives the simulated Thrust merge to the single-warp count)."""
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


def _warp_streams(w, E, first_subproblem_index=0):
    """Address streams (DMM model, oracle/dmm.py) of the w lanes of one warp of
    the unmodified Thrust serial merge (A | B forward in shared memory) on the
    oracle's labelling of a warp: d subproblems, T and switched T alternating,
    each thread's E outputs in the oracle's merge order."""
    d = gcd(w, E)
    patT, patS = wc.subproblem_label_patterns(w, E)
    labels = []
    for s in range(d):
        labels += list(patT if (first_subproblem_index + s) % 2 == 0 else patS)
    A = [o for o, l in enumerate(labels) if not l]
    B = [o for o, l in enumerate(labels) if l]
    smem = A + B
    streams, a, b = [], 0, 0
    for t in range(w):
        seg = labels[t * E:(t + 1) * E]
        nb = sum(seg)
        streams.append(dmm.serial_merge_addresses(smem, a, len(A) + b, E - nb, nb, E))
        a += E - nb
        b += nb
    return streams


def _simulate_warp_serial_merge(w, E, first_subproblem_index=0):
    return dmm.warp_instruction_conflicts(_warp_streams(w, E, first_subproblem_index), w)


def _lockstep_reads(w, E, streams):
    """Reads that land in bank w-E+s-1 at serial-merge step s = 2..E+1: the
    scan of the bottom E banks the proof of Theorem 8 counts (PAPER.md:300:
    'we count the number of bank conflicts in the last E shared memory banks';
    :255-259 the pure tuples 'aligned at the bottom E rows ... forced to
    perform a sequential scan of the bottom E banks')."""
    return sum(1 for s in range(2, E + 2) for st in streams if st[s] % w == (w - E + s - 1) % w)


@pytest.mark.parametrize("w", W_SET)
def test_theorem8_counts_the_lockstep_scan_of_the_bottom_banks(w):
    """With each mixed thread reading its x part first and its y part last
    (reading c9), the reads aligned with the bottom-E-bank scan number exactly
    Theorem 8 (combined) for every 1 < E <= w, for T-first and
    switched-first warps.  B-first (the round-1 reading) or y-first orders miss
    it for E > w/2 (e.g. w = 32, E = 19, 22..31)."""
    for E in range(2, w + 1):
        for f in (0, 1):
            assert _lockstep_reads(w, E, _warp_streams(w, E, f)) == wc.theorem8_warp(w, E), (E, f)


@pytest.mark.parametrize("w", W_SET)
def test_simulated_conflicts_at_least_theorem8(w):
    """Theorem 8 is what the construction guarantees ('we can align accesses
    that result in ...').  The simulated total (extra wavefronts
    + 1, reading c14) is >= Theorem 8 everywhere and equal in Case 1
    (E <= w/2), where every column ends with one aligned scan; in Case 2 the x
    parts the proof calls misaligned also meet each other in lockstep."""
    for E in range(2, w + 1):
        sim = _simulate_warp_serial_merge(w, E) + 1
        thm = wc.theorem8_warp(w, E)
        assert sim >= thm, (E, sim, thm)
        if E <= w / 2:
            assert sim == thm, (E, sim, thm)
        assert _simulate_warp_serial_merge(w, E, 1) + 1 == sim      # switched warp: mirror


def _best_path_gain(w, E, streams, t, a, b):
    """Best total step cost over all interleavings of lane t's a A-reads and
    b B-reads with the other lanes fixed (DP over the lattice path)."""
    others = [st for k, st in enumerate(streams) if k != t]
    steps = len(streams[0])
    per_step = []
    for s in range(steps):
        banks = {}
        for st in others:
            banks.setdefault(st[s] % w, set()).add(st[s])
        per_step.append(banks)

    def step_cost(s, x):
        banks = per_step[s]
        top = max((len(v) for v in banks.values()), default=0)
        here = banks.get(x % w, set())
        c = len(here) + (0 if x in here else 1)
        return max(top, c) - 1

    a0, b0 = streams[t][0], streams[t][1]
    fixed = step_cost(0, a0) + step_cost(1, b0)
    best = {}
    for i in range(a, -1, -1):
        for j in range(b, -1, -1):
            if i + j == E:
                best[(i, j)] = 0
                continue
            s = 2 + i + j
            opts = []
            if i < a:
                opts.append(step_cost(s, a0 + i + 1) + best[(i + 1, j)])
            if j < b:
                opts.append(step_cost(s, b0 + j + 1) + best[(i, j + 1)])
            best[(i, j)] = max(opts)
    return fixed + best[(0, 0)]


@pytest.mark.parametrize("E", [17, 19, 23, 26, 29, 31])
def test_interleaving_is_a_local_maximum(E):
    """No single mixed thread of the warp can raise the warp's simulated
    conflicts by reading its A and B members in another order (exhaustive over
    that thread's interleavings, the others fixed)."""
    w = 32
    streams = _warp_streams(w, E)
    total = dmm.warp_instruction_conflicts(streams, w)
    patT, _ = wc.subproblem_label_patterns(w, E)
    for t in range(w):
        seg = patT[t * E:(t + 1) * E]
        nb = int(seg.sum())
        if nb in (0, E):
            continue
        assert _best_path_gain(w, E, streams, t, E - nb, nb) == total, (E, t)


def test_theorem8_default_parameters():
    """The sort's defaults: keys (E, u) = (31, 128), pairs (11, 256) (bcf.h).
    Theorem 8 per warp: 526 (Case 2, r = 1) and 121 (Case 1)."""
    assert wc.theorem8_warp(32, 31) == 526
    assert wc.theorem8_warp(32, 11) == 121
    assert _lockstep_reads(32, 31, _warp_streams(32, 31)) == 526
    assert _simulate_warp_serial_merge(32, 31) + 1 >= 526


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
                                   (16, 64, 2 ** 13), (12, 64, 12 * 2 ** 9), (8, 128, 2 ** 13),
                                   (31, 128, 31 * 2 ** 10), (19, 64, 19 * 2 ** 9), (24, 64, 24 * 2 ** 9)])
def test_composition_hits_theorem8_at_every_regular_level(E, u, n):
    w = 32
    x = wc.worst_case_input(n, E, u, seed=1234)
    assert sorted(x.tolist()) == list(range(n))              # a permutation of ranks
    np.testing.assert_array_equal(x, wc.worst_case_input(n, E, u, seed=1234))  # deterministic
    # bottom-up simulation of the sort: runs of E first
    keys = x.astype(np.int64).copy()
    for s in range(0, n, E):
        keys[s:s + E] = np.sort(keys[s:s + E])
    warp = _simulate_warp_serial_merge(w, E)          # one warp of the pattern
    assert warp + 1 >= wc.theorem8_warp(w, E)
    regular_levels = 0
    for R in wc.merge_levels(n, E, u):
        keys, per_warp = _thrust_level_conflicts(keys, R, E, u, w)
        if per_warp:
            regular_levels += 1
            assert all(c == warp for c in per_warp), (R, set(per_warp))
    np.testing.assert_array_equal(keys, np.arange(n))
    assert regular_levels >= 3


def test_composition_ragged_sizes_are_permutations():
    for E, u in [(15, 64), (31, 128), (16, 256)]:
        for n in [0, 1, 14, 15, 16, 1000, 3841, 9999, 3 * 31 * 128 + 5]:
            x = wc.worst_case_input(n, E, u, seed=9)
            assert sorted(x.tolist()) == list(range(n))


def test_irregular_groups_have_exact_counts_and_random_pairs():
    """Ragged / sub-two-warp groups: exact |A| (the stable partition must fill
    the A child exactly), pairs (2k, 2k+1) one A and one B each, roughly half
    of them (B, A)."""
    n, E, u = 5000, 15, 64
    x = wc.worst_case_input(n, E, u, seed=3)
    # level R = E: groups of 2E; after sorting runs of E, each group's merge
    # takes exactly one element of each child run per output pair
    runs = [np.sort(x[s:s + E]) for s in range(0, n, E)]
    flips = 0
    pairs = 0
    for g in range(0, len(runs) - 1, 2):
        A, B = runs[g], runs[g + 1]
        merged = np.sort(np.concatenate([A, B]), kind="stable")
        src = np.isin(merged, B)
        assert src.sum() == len(B)
        for k in range(len(B)):
            assert src[2 * k] != src[2 * k + 1]
            flips += int(src[2 * k])
            pairs += 1
    assert 0.4 < flips / pairs < 0.6
