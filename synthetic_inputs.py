"""Seeded synthetic input generators shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the sorting method: only the counter-based
random stream (splitmix64) and the recipes that turn it into the workloads of
SURVEY.md §8(d) ("Concrete inputs").  Both the oracle (tests, bench's
cpu_baseline leg) and the product path (bench, GPU tests) draw their inputs from
here, so the two sides see bit-identical data without sharing method code.

Stream definition:
    h_i = mix64(seed + (i + 1) * 0x9E3779B97F4A7C15)            (mod 2^64)
    mix64(z): z ^= z >> 30; z *= 0xBF58476D1CE4E5B9;
              z ^= z >> 27; z *= 0x94D049BB133111EB; z ^= z >> 31
It is counter-based, so any slice [lo, hi) can be generated independently
(used for per-rank shards of a distributed input).

Recipes (the paper sorts "4-byte integers", §5; the others are
the north star's f32 / pairs configurations):
    uniform_u32      key = hi32(h_i)
    dup_u32          key = hi32(h_i) & 0xFFFF      (heavy duplicates: stability observable)
    uniform_f32      key = (h_i >> 40) * 2^-24     (uniform in [0, 1))
    special_f32      a mix of +-0, +-inf, NaN payloads, denormals and normals
    iota_u32         value = global index (pairs: values record input position)
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)

# Per-config seeds: seed = 0xB200_0000 + config_id.
SEED_BASE = 0xB200_0000


def config_seed(config_id: int) -> int:
    return SEED_BASE + int(config_id)


def _mix64(z: np.ndarray) -> np.ndarray:
    z = z ^ (z >> np.uint64(30))
    z = z * M1
    z = z ^ (z >> np.uint64(27))
    z = z * M2
    z = z ^ (z >> np.uint64(31))
    return z


def splitmix64(seed: int, lo: int, hi: int, chunk: int = 1 << 22) -> np.ndarray:
    """h_i for i in [lo, hi) as uint64 (chunked to bound temporaries)."""
    n = max(0, hi - lo)
    out = np.empty(n, dtype=np.uint64)
    s = np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
    with np.errstate(over="ignore"):
        for c0 in range(0, n, chunk):
            c1 = min(n, c0 + chunk)
            i = np.arange(lo + c0 + 1, lo + c1 + 1, dtype=np.uint64)
            out[c0:c1] = _mix64(s + i * GOLDEN)
    return out


def uniform_u32(n: int, seed: int, lo: int = 0) -> np.ndarray:
    return (splitmix64(seed, lo, lo + n) >> np.uint64(32)).astype(np.uint32)


def dup_u32(n: int, seed: int, lo: int = 0, mask: int = 0xFFFF) -> np.ndarray:
    return uniform_u32(n, seed, lo) & np.uint32(mask)


def uniform_f32(n: int, seed: int, lo: int = 0) -> np.ndarray:
    h = splitmix64(seed, lo, lo + n) >> np.uint64(40)
    return (h.astype(np.float64) * (2.0 ** -24)).astype(np.float32)


def iota_u32(n: int, lo: int = 0) -> np.ndarray:
    return np.arange(lo, lo + n, dtype=np.uint64).astype(np.uint32)


_SPECIAL_BITS = np.array(
    [
        0x00000000,  # +0
        0x80000000,  # -0
        0x7F800000,  # +inf
        0xFF800000,  # -inf
        0x7FC00000,  # +qNaN
        0xFFC00000,  # -qNaN
        0x7F800001,  # +sNaN payload 1
        0xFF800001,  # -sNaN payload 1
        0x7FFFFFFF,  # +NaN max payload
        0xFFFFFFFF,  # -NaN max payload
        0x00000001,  # +min denormal
        0x80000001,  # -min denormal
        0x007FFFFF,  # +max denormal
        0x807FFFFF,  # -max denormal
        0x00800000,  # +min normal
        0x80800000,  # -min normal
        0x7F7FFFFF,  # +max finite
        0xFF7FFFFF,  # -max finite
        0x3F800000,  # +1
        0xBF800000,  # -1
    ],
    dtype=np.uint32,
)


def special_f32_bits(n: int, seed: int) -> np.ndarray:
    """Bit patterns: half drawn from the special set, half arbitrary 32-bit words
    (every 32-bit word is a valid float bit pattern, including NaNs)."""
    h = splitmix64(seed, 0, n)
    pick = (h & np.uint64(1)).astype(bool)
    idx = ((h >> np.uint64(8)) % np.uint64(len(_SPECIAL_BITS))).astype(np.int64)
    raw = (h >> np.uint64(32)).astype(np.uint32)
    return np.where(pick, _SPECIAL_BITS[idx], raw).astype(np.uint32)


# ---------------------------------------------------------------------------
# Device-side twin of the same stream (torch, for large benchmark inputs).
# int64 arithmetic in torch wraps modulo 2^64 (two's complement), so the
# products are bit-identical; right shifts are made logical with a mask.
# ---------------------------------------------------------------------------

def _to_i64(x: int) -> int:
    x &= 0xFFFFFFFFFFFFFFFF
    return x - (1 << 64) if x >= (1 << 63) else x


def _lsr(t, s: int):
    import torch  # noqa: F401

    return (t >> s) & ((1 << (64 - s)) - 1)


def splitmix64_torch(seed: int, lo: int, hi: int, device, chunk: int = 1 << 24):
    import torch

    n = max(0, hi - lo)
    out = torch.empty(n, dtype=torch.int64, device=device)
    g = _to_i64(int(GOLDEN))
    m1 = _to_i64(int(M1))
    m2 = _to_i64(int(M2))
    s = _to_i64(seed)
    for c0 in range(0, n, chunk):
        c1 = min(n, c0 + chunk)
        z = torch.arange(lo + c0 + 1, lo + c1 + 1, dtype=torch.int64, device=device)
        z = z * g + s
        z = z ^ _lsr(z, 30)
        z = z * m1
        z = z ^ _lsr(z, 27)
        z = z * m2
        z = z ^ _lsr(z, 31)
        out[c0:c1] = z
    return out


def uniform_u32_torch(n: int, seed: int, device, lo: int = 0):
    """Same values as uniform_u32, as an int32 tensor holding the u32 bit pattern."""
    import torch

    h = splitmix64_torch(seed, lo, lo + n, device)
    hi = _lsr(h, 32)
    return (hi - ((hi >= (1 << 31)).to(torch.int64) << 32)).to(torch.int32)


def uniform_f32_torch(n: int, seed: int, device, lo: int = 0):
    """Same values as uniform_f32 (exact: 24-bit integers times 2^-24), as a float32 tensor."""
    import torch

    h = splitmix64_torch(seed, lo, lo + n, device)
    return _lsr(h, 40).to(torch.float32) * (2.0 ** -24)


def dup_u32_torch(n: int, seed: int, device, lo: int = 0, mask: int = 0xFFFF):
    """Same values as dup_u32, as an int32 tensor."""
    return uniform_u32_torch(n, seed, device, lo) & mask


def iota_u32_torch(n: int, device, lo: int = 0):
    """Same values as iota_u32 (for n + lo <= 2^31), as an int32 tensor."""
    import torch

    return torch.arange(lo, lo + n, dtype=torch.int64, device=device).to(torch.int32)
