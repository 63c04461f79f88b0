"""oracle/addrmap.py -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper's shared-memory address maps and its load-balanced dual subsequence
gather, written out step by step in the paper's notation (w banks, E items per
thread, d = GCD(w, E), u threads per block).

    pi   : reverse the B list                       PAPER.md:152-160 §3.1
    rho  : circular shift of partitions of wE/d     PAPER.md:162-211 §3.2, :219 §3.3
    Alg. 1 DUAL-SUBSEQUENCE-GATHER

Reading adopted: partition l is
rotated RIGHT by (l mod d) positions, i.e. the element at offset x of the
partition lands at offset (x + l mod d) mod P.  This is the direction pinned by
Figure 3 (tests/golden/fig3_w9_E6.txt).
"""
from __future__ import annotations

from math import gcd


def d_of(w: int, E: int) -> int:
    """d = GCD(w, E)  (Table 1)."""
    return gcd(w, E)


def partition_size(w: int, E: int) -> int:
    """P = wE/d elements per rho-partition."""
    return w * E // d_of(w, E)


def rho(k: int, w: int, E: int) -> int:
    """Logical index k -> physical shared-memory index.

    Partition l = floor(k / P) is circularly shifted by (l mod d) positions
    ("we align the accesses to elements in the l-th partition
    by performing a circular shift of l locations"; extended to a thread block
    with shift l mod d).  For d = 1 this is the identity.
    """
    d = d_of(w, E)
    P = partition_size(w, E)
    l = k // P
    x = k - l * P
    return l * P + (x + (l % d)) % P


def rho_inv(p: int, w: int, E: int) -> int:
    d = d_of(w, E)
    P = partition_size(w, E)
    l = p // P
    y = p - l * P
    return l * P + (y - (l % d)) % P


def pi_B(y: int, NA: int, NB: int) -> int:
    """Logical position of B[y] after reversing B behind A:
    B[y] sits at (NA + NB - 1) - y."""
    return NA + NB - 1 - y


def round_of(k: int, E: int) -> int:
    """After rho, the element at logical index k is read in round k mod E
    (PAPER.md:211)."""
    return k % E


def gather_indices(a_i: int, b_i: int, nA_i: int, nB_i: int, NA: int, NB: int,
                   w: int, E: int):
    """Alg. 1 for one thread: the physical shared-memory
    index read in each round j = 0..E-1, and which element it is.

    Returns a list of (phys_idx, ('A', x) | ('B', y) | None) per round.  A
    round with no element (|A_i| + |B_i| < E, a ragged tile, SURVEY.md §8(c)
    c12) reads nothing and is reported as (None, None).
    """
    k = a_i % E                                          # line 3
    out = []
    for j in range(E):                                   # line 4
        ia = (j - k) % E
        if ia < nA_i:                                    # line 5
            idx = rho(ia + a_i, w, E)                    # line 6
            out.append((idx, ("A", a_i + ia)))
        else:
            ib = (k - j - 1) % E                         # line 8
            if ib < nB_i:
                idx = rho(pi_B(ib + b_i, NA, NB), w, E)
                out.append((idx, ("B", b_i + ib)))
            else:
                out.append((None, None))
    return out


def layout_owner_grid(splits, NA: int, NB: int, w: int, E: int, reverse_B=True,
                      use_rho=True):
    """Physical shared-memory cell -> owning thread, for a warp/block whose
    threads take (a_i, b_i, |A_i|, |B_i|) = splits[i].  This is the picture the
    paper draws in Figs. 2, 3, 7, 8 (column-major, w rows = banks)."""
    T = NA + NB
    cells = [None] * T
    for t, (a, b, na, nb) in enumerate(splits):
        for x in range(a, a + na):
            k = x
            cells[rho(k, w, E) if use_rho else k] = t
        for y in range(b, b + nb):
            k = pi_B(y, NA, NB) if reverse_B else NA + y
            cells[rho(k, w, E) if use_rho else k] = t
    return cells
