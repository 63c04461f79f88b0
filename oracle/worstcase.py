"""oracle/worstcase.py -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper's worst-case inputs for the unmodified Thrust mergesort, Section 4
(PAPER.md:221-344), written step by step in the paper's notation, plus the
multi-level composition the paper defers to [8] (DESIGN.md
"Readings").

Per subproblem of w/d threads and wE/d outputs:
    w = qE + r  (Euclid, Lemma 9)
    s_i = i (r/d) mod (E/d),  x_i = (E/d - s_i) d,  y_i = s_i d,   i = 1..E/d-1
    S: a_i = x_i if i even else y_i;  b_i = x_i if i odd else y_i
    T: steps (1)-(3), PAPER.md:261-266 (garbled text read per SURVEY.md c7)
Theorem 8 (combined :342).

Order inside a mixed thread (reading c9): the thread of S-tuple i
reads its x_i part first and its y_i part last.  The proof
counts conflicts in the bottom E banks: every column of w words is
x_i | y_{i+1} | pure tuples (x_i + y_{i+1} = r or E + r, Lemma 7), so a y part
that ends the column at bank w-1 is in lockstep with the pure threads' scan of
banks w-E..w-1 only if it is read LAST, and an x part (banks 0..x_i-1, the
"(x_i - r) misaligned elements") can never be.  Under this order the number of
reads that land in the scanned bank w-E+s-1 at serial-merge step s is exactly
Theorem 8 for every 1 < E <= w (tests/test_oracle_worstcase.py); the total
conflicts are >= Theorem 8, because the x parts, which the proof does not
count, are read in lockstep with one another.

Multi-level composition (reading c10): start from the sorted output 0..n-1 and
walk the merge levels top-down; every REGULAR merge group (full, and its run
size a multiple of wE, i.e. at least two warps of outputs) labels each output
A or B from T (even subproblem index) / switched T (odd index).  Every other
group (block-sort levels with groups of less than two warps, ragged tails)
gets a random exact-count labelling that is a closed form of the position: the
first 2 nb outputs form pairs (2k, 2k+1), pair k is (B, A) if the top bit of a
counter-based stream word at the pair's absolute index is set and (A, B)
otherwise, and the remaining na - nb outputs are A.  Labelled positions are
stable-partitioned into the two child runs.  At the bottom each run of E (one
thread's items) is shuffled (Fisher-Yates driven by the same counter-based
stream) because thread-local order is irrelevant.
"""
from __future__ import annotations

from math import gcd

import numpy as np

MASK64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15
LEVEL_SALT = 0xD1B54A32D192ED03
SHUFFLE_SALT = 0x2545F4914F6CDD1D


def mix64(z: int) -> int:
    z &= MASK64
    z ^= z >> 30
    z = (z * 0xBF58476D1CE4E5B9) & MASK64
    z ^= z >> 27
    z = (z * 0x94D049BB133111EB) & MASK64
    z ^= z >> 31
    return z


def _mix64_np(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = z ^ (z >> np.uint64(30))
        z = z * np.uint64(0xBF58476D1CE4E5B9)
        z = z ^ (z >> np.uint64(27))
        z = z * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def stream_np(seed: int, positions: np.ndarray) -> np.ndarray:
    """h(p) = mix64(seed + (p + 1) * GOLDEN) for an array of positions."""
    with np.errstate(over="ignore"):
        z = np.uint64(seed & MASK64) + (positions.astype(np.uint64) + np.uint64(1)) * np.uint64(GOLDEN)
    return _mix64_np(z)


# ---------------------------------------------------------------------------
# Section 4: S, T, Theorem 8
# ---------------------------------------------------------------------------

def euclid(w: int, E: int):
    """w = qE + r, 0 <= r < E (Lemma 9 as used at PAPER.md:227)."""
    return w // E, w % E


def S_sequence(w: int, E: int):
    """[(i, s_i, x_i, y_i, a_i, b_i)] for i = 1..E/d-1."""
    d = gcd(w, E)
    q, r = euclid(w, E)
    Ed, rd = E // d, r // d
    out = []
    for i in range(1, Ed):
        s = (i * rd) % Ed
        x = (Ed - s) * d
        y = s * d
        a = x if i % 2 == 0 else y
        b = x if i % 2 == 1 else y
        out.append((i, s, x, y, a, b))
    return out


def T_sequence(w: int, E: int):
    """[(a, b)] of T_sequence_indexed (the S index dropped)."""
    return [(a, b) for (a, b, _) in T_sequence_indexed(w, E)]


def T_sequence_indexed(w: int, E: int):
    """The tuple sequence T of Section 4, |T| = w/d.

    Each entry is (a, b, i): i is the index of the S-tuple it came from, or 0
    for an inserted pure tuple ((E, 0) / (0, E)).
    E | w (d = E, S empty) is not spelled out by the paper; reading c8 takes
    T = q tuples (E, 0)."""
    assert 1 < E <= w
    d = gcd(w, E)
    q, r = euclid(w, E)
    Ed = E // d
    if Ed == 1:
        return [(E, 0, 0)] * q
    S = S_sequence(w, E)
    x = {i: xi for (i, _, xi, _, _, _) in S}
    y = {i: yi for (i, _, _, yi, _, _) in S}
    ab = {i: (a, b) for (i, _, _, _, a, b) in S}
    T = []
    # (1) (a_1, b_1) = (y_1, x_1) = (r, E - r), followed by q tuples of (E, 0)
    T.append((y[1], x[1], 1))
    T.extend([(E, 0, 0)] * q)
    # (2) for i = 1..E/d-2: insert (a_{i+1}, b_{i+1}), then q or q-1 pure tuples
    for i in range(1, Ed - 1):
        T.append(ab[i + 1] + (i + 1,))
        pure = (E, 0, 0) if i % 2 == 0 else (0, E, 0)
        if x[i] + y[i + 1] == r:
            T.extend([pure] * q)
        else:
            assert x[i] + y[i + 1] == E + r  # Lemma 7
            T.extend([pure] * (q - 1))
    # (3) q tuples of (E, 0) if E/d - 1 is even, else (0, E)
    T.extend([(E, 0, 0) if (Ed - 1) % 2 == 0 else (0, E, 0)] * q)
    assert len(T) == w // d
    return T


def switched(T):
    """the symmetric case switches the tuple values."""
    return [(b, a) for (a, b) in T]


def theorem8_subproblem(w: int, E: int) -> float:
    """Theorem 8: bank conflicts for one subproblem."""
    d = gcd(w, E)
    q, r = euclid(w, E)
    if E <= w / 2:
        return E * E / d
    return 0.5 * (E * E / d + 2 * E * r / d + E - r * r / d - r)


def theorem8_warp(w: int, E: int) -> float:
    """Combined over the d subproblems of a warp."""
    d = gcd(w, E)
    q, r = euclid(w, E)
    if 1 < E <= w / 2:
        return float(E * E)
    return 0.5 * (E * E + 2 * E * r + E * d - r * r - r * d)


def warp_thread_tuples(w: int, E: int, first_subproblem_index: int = 0):
    """(a_i, b_i) for the w threads of one warp: its d subproblems take T and
    switched T alternately by global subproblem index."""
    d = gcd(w, E)
    T = T_sequence(w, E)
    out = []
    for s in range(d):
        seq = T if (first_subproblem_index + s) % 2 == 0 else switched(T)
        out.extend(seq)
    return out


# ---------------------------------------------------------------------------
# Multi-level composition (reading c10)
# ---------------------------------------------------------------------------

def thread_labels(a: int, b: int, i: int, switched_: bool):
    """Labels (True = B) of one thread's E outputs in merge order (reading c9).

    S-tuple i is (a_i, b_i) = (y_i, x_i) for odd i and (x_i, y_i) for even i
    (PAPER.md:229-231), so its x part is the B part under T for odd i and the
    A part for even i; a switched subproblem swaps the lists.
    The x part is read first, the y part last.  Pure tuples have one list."""
    if i == 0:
        return [True] * b + [False] * a
    x_is_B = (i % 2 == 1) != switched_
    if x_is_B:
        return [True] * b + [False] * a
    return [False] * a + [True] * b


def subproblem_label_patterns(w: int, E: int):
    """Label (True = B) of each output position of a T-subproblem and of a
    switched-T subproblem."""
    pT, pS = [], []
    for (a, b, i) in T_sequence_indexed(w, E):
        pT.extend(thread_labels(a, b, i, False))
        pS.extend(thread_labels(b, a, i, True))
    return np.array(pT, dtype=bool), np.array(pS, dtype=bool)


def merge_levels(n: int, E: int, u: int):
    """Child run sizes R of every merge level of the pairwise mergesort, bottom
    up: block-sort levels E, 2E, ..., uE/2 (merges inside a tile of uE), then
    global passes T, 2T, ... while R < n."""
    levels = []
    R = E
    tile = u * E
    while R < tile and R < n:
        levels.append(R)
        R *= 2
    R = tile
    while R < n:
        levels.append(R)
        R *= 2
    return levels


def worst_case_input(n: int, E: int, u: int, seed: int, w: int = 32) -> np.ndarray:
    """A permutation of 0..n-1 that drives the unmodified Thrust merge to the
    Theorem 8 conflict count at every regular merge level."""
    if n == 0:
        return np.zeros(0, dtype=np.uint32)
    vals = np.arange(n, dtype=np.int64)
    d = gcd(w, E)
    sp = w * E // d
    patT, patS = subproblem_label_patterns(w, E)
    pos = np.arange(n, dtype=np.int64)
    for R in reversed(merge_levels(n, E, u)):
        g = pos // (2 * R)
        p = pos - g * 2 * R
        g0 = g * 2 * R
        m = np.minimum(2 * R, n - g0)
        na = np.minimum(R, m)
        label_B = np.zeros(n, dtype=bool)
        regular = (m == 2 * R) & (R % (w * E) == 0)
        if regular.any():
            pr = p[regular]
            sub = pr // sp
            off = pr - sub * sp
            label_B[regular] = np.where(sub % 2 == 0, patT[off], patS[off])
        irr = ~regular
        if irr.any():
            # pairs (2k, 2k+1) of the first 2 nb outputs: (B, A) if the top bit
            # of h(absolute pair index) is set, else (A, B); the rest are A
            seed_l = (seed + R * LEVEL_SALT) & MASK64
            pi = p[irr]
            nb = (m - na)[irr]
            pair_abs = (g0[irr] + pi - (pi & 1)) // 2
            bit = (stream_np(seed_l, pair_abs) >> np.uint64(63)).astype(np.int64)
            label_B[irr] = (pi < 2 * nb) & (((pi & 1) ^ bit) == 1)
        # stable partition of every group: the A-labelled outputs, in order,
        # fill the A child [g0, g0 + na), the B-labelled ones the B child
        isA = ~label_B
        cumA = np.cumsum(isA) - isA                      # A labels before p
        cumB = np.cumsum(label_B) - label_B              # B labels before p
        rankA = cumA - cumA[g0]
        rankB = cumB - cumB[g0]
        dest = np.where(isA, g0 + rankA, g0 + na + rankB)
        nxt = np.empty_like(vals)
        nxt[dest] = vals
        vals = nxt
    # bottom: shuffle every run of E (one thread's items); Fisher-Yates with
    # j = floor(hi32(h) * (i + 1) / 2^32)
    seed_s = (seed + SHUFFLE_SALT) & MASK64
    h = stream_np(seed_s, pos)
    hi = (h >> np.uint64(32)).astype(np.uint64)
    run0 = (pos // E) * E
    runlen = np.minimum(E, n - run0)
    i_in = pos - run0
    for i in range(E - 1, 0, -1):
        sel = (i_in == i) & (runlen > i)
        if not sel.any():
            continue
        src = pos[sel]
        j = ((hi[sel] * np.uint64(i + 1)) >> np.uint64(32)).astype(np.int64)
        dst = run0[sel] + j
        a = vals[src].copy()
        vals[src] = vals[dst]
        vals[dst] = a
    return vals.astype(np.uint32)
