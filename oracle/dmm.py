"""oracle/dmm.py -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Distributed Memory Machine cost model of shared memory (PAPER.md:53, :69,
:95-99 §2): w banks, bank(i) = i mod w; one warp instruction costs as many
"wavefronts" as the largest number of DISTINCT addresses that fall in one bank
(footnote 4: lanes reading the same address do not conflict).
ncu reports conflicts = wavefronts - 1 per instruction.

Also the Thrust/CUB serial merge the paper's worst case targets:
each thread, after its merge-path split, walks A_i and B_i in shared memory
reading one element per output ("the naive (sequential) processing of A_i and
B_i by the i-th thread directly in shared memory").
"""
from __future__ import annotations


def wavefronts(addrs, w: int = 32) -> int:
    """addrs: one word address per lane, None for an inactive lane."""
    per_bank = {}
    for a in addrs:
        if a is None:
            continue
        per_bank.setdefault(a % w, set()).add(a)
    if not per_bank:
        return 0
    return max(len(s) for s in per_bank.values())


def conflicts(addrs, w: int = 32) -> int:
    wf = wavefronts(addrs, w)
    return max(0, wf - 1)


def serial_merge_addresses(keys_smem, a_beg, b_beg, nA, nB, E):
    """Address stream of one thread of the unmodified Thrust serial merge
    (A stored at [0, NA), B stored right behind it, NOT reversed).

    keys_smem: the tile as stored in shared memory; a_beg/b_beg are shared
    memory positions of A_i[0] and B_i[0].  Returns E + 2 addresses: the two
    initial loads, then one load per output (the element that replaces the one
    just consumed).  Ties go to A ("take B only if B < A").
    """
    a_end = a_beg + nA
    b_end = b_beg + nB
    addrs = [a_beg, b_beg]
    k1 = keys_smem[a_beg] if a_beg < len(keys_smem) else None
    k2 = keys_smem[b_beg] if b_beg < len(keys_smem) else None
    for _ in range(E):
        take_b = (b_beg < b_end) and ((a_beg >= a_end) or (k2 < k1))
        if take_b:
            b_beg += 1
            addrs.append(b_beg)
            k2 = keys_smem[b_beg] if b_beg < len(keys_smem) else None
        else:
            a_beg += 1
            addrs.append(a_beg)
            k1 = keys_smem[a_beg] if a_beg < len(keys_smem) else None
    return addrs


def warp_instruction_conflicts(per_lane_streams, w: int = 32):
    """Sum of (wavefronts - 1) over the instructions of a warp whose lanes issue
    the given equal-length address streams in lockstep (PAPER.md footnote 2)."""
    if not per_lane_streams:
        return 0
    steps = len(per_lane_streams[0])
    total = 0
    for s in range(steps):
        total += conflicts([st[s] for st in per_lane_streams], w)
    return total
