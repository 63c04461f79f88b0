"""Pins for oracle/setops_oracle.c (set operations with multiset semantics,
ISO C++ [alg.set.operations]; the paper's "parallel scan of a pair of
arrays") against an independent statement of the same
definition: per-key copy counts from collections.Counter, and, for the source
indices, the "first"/"last" copies of each key's run written with Python
lists; plus brute force over all small inputs and the library identities."""
import itertools
from collections import Counter

import numpy as np
import pytest

import oracle


def _expected(op, a, b):
    ca, cb = Counter(a.tolist()), Counter(b.tolist())
    keys, srcs = [], []
    for x in sorted(set(ca) | set(cb)):
        ia = [i for i, v in enumerate(a.tolist()) if v == x]      # A's copies of x, in order
        ib = [j for j, v in enumerate(b.tolist()) if v == x]
        m, n = len(ia), len(ib)
        if op == "union":
            take = [(i, 0) for i in ia] + [(j, 1) for j in ib[m:]]                # last n - m of B
        elif op == "intersection":
            take = [(i, 0) for i in ia[:min(m, n)]]
        elif op == "difference":
            take = [(i, 0) for i in ia[n:]] if m > n else []                      # last m - n of A
        else:
            take = [(i, 0) for i in ia[n:]] if m > n else [(j, 1) for j in ib[m:]]
        for idx, fromb in take:
            keys.append(x)
            srcs.append((0x80000000 | idx) if fromb else idx)
    return np.array(keys, dtype=np.uint32), np.array(srcs, dtype=np.uint32)


OPS = ["union", "intersection", "difference", "symmetric_difference"]


@pytest.mark.parametrize("op", OPS)
def test_brute_force_small_multisets(op):
    """Every pair of sorted sequences over {0, 1, 2} with lengths 0..4."""
    seqs = [np.array(sorted(s), dtype=np.uint32) for n in range(5) for s in itertools.product(range(3), repeat=n)]
    seqs = list({tuple(s.tolist()): s for s in seqs}.values())
    for a in seqs:
        for b in seqs:
            k, s = oracle.set_op_u32(op, a, b)
            ek, es = _expected(op, a, b)
            np.testing.assert_array_equal(k, ek)
            np.testing.assert_array_equal(s, es)


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("mask", [0x7, 0xFF, 0xFFFFFFFF])
def test_random_against_counter_definition(op, mask):
    rng = np.random.default_rng(mask % 1000 + len(op))
    for _ in range(20):
        a = np.sort(rng.integers(0, 1 << 32, size=rng.integers(0, 300), dtype=np.uint64).astype(np.uint32) & mask)
        b = np.sort(rng.integers(0, 1 << 32, size=rng.integers(0, 300), dtype=np.uint64).astype(np.uint32) & mask)
        k, s = oracle.set_op_u32(op, a, b)
        ek, es = _expected(op, a, b)
        np.testing.assert_array_equal(k, ek)
        np.testing.assert_array_equal(s, es)


def test_identities():
    """|A u B| + |A n B| = |A| + |B|; (A - B) ++ (A n B) is A as a multiset;
    symmetric difference = (A - B) u (B - A); numpy's set routines on sets."""
    rng = np.random.default_rng(5)
    a = np.sort(rng.integers(0, 50, 1000).astype(np.uint32))
    b = np.sort(rng.integers(0, 50, 700).astype(np.uint32))
    u, _ = oracle.set_op_u32("union", a, b)
    i, _ = oracle.set_op_u32("intersection", a, b)
    d, _ = oracle.set_op_u32("difference", a, b)
    d2, _ = oracle.set_op_u32("difference", b, a)
    x, _ = oracle.set_op_u32("symmetric_difference", a, b)
    assert u.size + i.size == a.size + b.size
    np.testing.assert_array_equal(np.sort(np.concatenate([d, i])), a)
    np.testing.assert_array_equal(x, np.sort(np.concatenate([d, d2])))
    # on sets (no duplicates) the operations are numpy's
    sa, sb = np.unique(a), np.unique(b)
    np.testing.assert_array_equal(oracle.set_op_u32("union", sa, sb)[0], np.union1d(sa, sb))
    np.testing.assert_array_equal(oracle.set_op_u32("intersection", sa, sb)[0], np.intersect1d(sa, sb))
    np.testing.assert_array_equal(oracle.set_op_u32("difference", sa, sb)[0], np.setdiff1d(sa, sb))
    np.testing.assert_array_equal(oracle.set_op_u32("symmetric_difference", sa, sb)[0], np.setxor1d(sa, sb))
