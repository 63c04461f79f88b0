"""Pins for oracle/sort_oracle.c against things other than itself:
library stable sorts (numpy, Python's sorted), brute force over all
permutations / all small words, and the IEEE 754 totalOrder clauses."""
import itertools
import struct

import numpy as np
import pytest

import oracle
import synthetic_inputs as si


SIZES = [0, 1, 2, 3, 14, 15, 16, 17, 255, 256, 3839, 3840, 3841, 4095, 4096, 4097, 10007, 65536]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("kind", ["uniform", "dup", "sorted", "reversed", "equal"])
def test_u32_matches_numpy_stable(n, kind):
    seed = si.config_seed(0) + n
    if kind == "uniform":
        x = si.uniform_u32(n, seed)
    elif kind == "dup":
        x = si.dup_u32(n, seed, mask=0x7)
    elif kind == "sorted":
        x = np.sort(si.uniform_u32(n, seed))
    elif kind == "reversed":
        x = np.sort(si.uniform_u32(n, seed))[::-1].copy()
    else:
        x = np.full(n, 0xFFFFFFFF, dtype=np.uint32)
    got = oracle.sort_u32(x)
    np.testing.assert_array_equal(got, np.sort(x, kind="stable"))


@pytest.mark.parametrize("n", [0, 1, 5, 300, 4097, 50000])
def test_pairs_stable_matches_numpy_argsort(n):
    k = si.dup_u32(n, si.config_seed(3) + n, mask=0xF)
    v = si.iota_u32(n)
    ko, vo = oracle.sort_pairs_u32(k, v)
    perm = np.argsort(k, kind="stable")
    np.testing.assert_array_equal(ko, k[perm])
    np.testing.assert_array_equal(vo, v[perm])


def test_brute_force_all_permutations():
    for n in range(0, 8):
        for p in itertools.permutations(range(n)):
            x = np.array(p, dtype=np.uint32)
            assert list(oracle.sort_u32(x)) == sorted(p)


def test_brute_force_stability_all_words():
    """All words over {0,1,2} up to length 8, values = index: the oracle must
    equal Python's stable sorted() (a library routine)."""
    for n in range(0, 9):
        for word in itertools.product((0, 1, 2), repeat=n):
            k = np.array(word, dtype=np.uint32)
            v = np.arange(n, dtype=np.uint32)
            ko, vo = oracle.sort_pairs_u32(k, v)
            exp = sorted(range(n), key=lambda i: word[i])
            assert list(vo) == exp
            assert list(ko) == [word[i] for i in exp]


def test_u32_extremes():
    x = np.array([0xFFFFFFFF, 0, 0x80000000, 0x7FFFFFFF, 1, 0xFFFFFFFE], dtype=np.uint32)
    assert list(oracle.sort_u32(x)) == sorted(int(a) for a in x)


# ---- f32 totalOrder -------------------------------------------------------

# IEEE 754-2008 §5.10 totalOrder, written out by hand as an ordered list of
# bit patterns (negative NaNs by descending payload, -inf, negative numbers,
# -0, +0, positive numbers, +inf, positive NaNs by ascending payload).
TOTAL_ORDER_EXPECTED = [
    0xFFFFFFFF,  # -NaN, max payload
    0xFFC00000,  # -qNaN
    0xFF800001,  # -sNaN payload 1
    0xFF800000,  # -inf
    0xFF7FFFFF,  # -max finite
    0xBF800000,  # -1
    0x80800000,  # -min normal
    0x807FFFFF,  # -max denormal
    0x80000001,  # -min denormal
    0x80000000,  # -0
    0x00000000,  # +0
    0x00000001,  # +min denormal
    0x007FFFFF,  # +max denormal
    0x00800000,  # +min normal
    0x3F800000,  # +1
    0x7F7FFFFF,  # +max finite
    0x7F800000,  # +inf
    0x7F800001,  # +sNaN payload 1
    0x7FC00000,  # +qNaN
    0x7FFFFFFF,  # +NaN, max payload
]


def test_f32_total_order_special_values():
    exp = np.array(TOTAL_ORDER_EXPECTED, dtype=np.uint32)
    rng = np.random.default_rng(7)
    for _ in range(20):
        x = rng.permutation(np.repeat(exp, 3))
        np.testing.assert_array_equal(oracle.sort_f32_bits(x), np.repeat(exp, 3))
    for i, a in enumerate(TOTAL_ORDER_EXPECTED):
        for j, b in enumerate(TOTAL_ORDER_EXPECTED):
            assert oracle.f32_total_less(a, b) == (i < j)


@pytest.mark.parametrize("n", [1, 100, 4096, 65536])
def test_f32_non_nan_matches_numeric_sort(n):
    """For non-NaN values with no zeros, totalOrder is numeric order: pin
    against numpy's float sort."""
    x = si.uniform_f32(n, si.config_seed(2) + n) * np.float32(4.0) - np.float32(2.0)
    x = x[x != 0]
    bits = x.view(np.uint32)
    got = oracle.sort_f32_bits(bits).view(np.float32)
    np.testing.assert_array_equal(got, np.sort(x, kind="stable"))


def test_f32_random_bit_patterns_against_key_sort():
    """Every 32-bit word is a float.  Pin: Python's stable sorted() with a key
    built from struct-unpacked (sign, exponent, mantissa) fields."""
    bits = si.special_f32_bits(20000, si.config_seed(2))

    def key(b):
        f = struct.unpack("<f", struct.pack("<I", int(b)))[0]
        sign = int(b) >> 31
        isnan = f != f
        mag = int(b) & 0x7FFFFFFF
        if sign == 0:
            return (1, 1 if isnan else 0, mag)
        return (0, 0 if isnan else 1, -mag)

    exp = sorted((int(b) for b in bits), key=key)
    assert list(oracle.sort_f32_bits(bits)) == exp


@pytest.mark.parametrize("n", [0, 1, 7, 1000, 100003, 1 << 20])
def test_oracle_matches_cpu_baselines(n):
    """The oracle against the library routine std::stable_sort and the
    parallel mergesort baseline."""
    x = si.uniform_u32(n, 99 + n) & np.uint32(0xFFFF if n % 2 else 0xFFFFFFFF)
    exp = oracle.sort_u32(x)
    np.testing.assert_array_equal(oracle.std_stable_sort_u32(x), exp)
    for th in (1, 3, 8):
        np.testing.assert_array_equal(oracle.parallel_mergesort_u32(x, th), exp)
