"""Distributed sort across the GPUs of one node.

One process per GPU.  Every rank holds a shard of keys (optionally values):
  1. local CF mergesort (bcf_sort_u32 / bcf_sort_pairs_u32), no communication;
  2. exact splitters: for targets k_t = floor(t N / p), t = 1..p-1, a k-ary
     bisection of the 32-bit key space finds the smallest key v_t with
     sum_r #(keys_r <= v_t) >= k_t; each round every rank counts with
     bcf_split_counts_u32 (device binary searches) and one all_reduce(SUM)
     combines the counts;
  3. equal keys at the cut are consumed in rank order (stable): rank r sends
     lt_r(v_t) + min(eq_r(v_t), max(0, k_t - L_t - sum_{r'<r} eq_r'(v_t)))
     keys below cut t, so rank r ends with exactly positions
     [k_r, k_{r+1}) of the global stable order;
  4. all_to_all_single exchanges the buckets (NCCL over NVLink / NVSwitch);
  5. bcf_merge_runs_u32 merges the p received runs in source-rank order
     (ties to the lower rank) with the CF merge kernel.

The local operations are injectable (`ops`) so the host logic can be tested
with the gloo backend on CPU; the default ops are the CUDA library and raise
without a GPU -- there is no CPU fallback in the product path.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

KEY_SPACE = 1 << 32
PIVOTS_PER_TARGET = 63  # (63+1)-ary search: 32 bits in 6 rounds


class CudaOps:
    """Local phases on the GPU through the C ABI."""

    def __init__(self, params=None):
        import paper_conf_spaa_berneys25_b200 as bcf

        self.bcf = bcf
        self.params = params

    def sort(self, keys, values=None):
        if values is None:
            return self.bcf.sort(keys, params=self.params), None
        return self.bcf.sort_pairs(keys, values, params=self.params)

    def split_counts(self, sorted_keys, pivots_u32: np.ndarray):
        import torch

        piv = torch.from_numpy(pivots_u32.astype(np.uint32).view(np.int32)).to(sorted_keys.device)
        lt, le = self.bcf.split_counts(sorted_keys, piv)
        return lt, le

    def merge_runs(self, keys, offsets, values=None):
        return self.bcf.merge_runs(keys, offsets, values=values, params=self.params) if values is not None \
            else (self.bcf.merge_runs(keys, offsets, params=self.params), None)


@dataclass
class DistStats:
    rounds: int = 0
    send_counts: list | None = None
    recv_counts: list | None = None
    pivots: list | None = None


def _staged(group) -> bool:
    """gloo cannot run collectives on CUDA tensors: stage them through host
    copies (a correctness path for the world-size-2 test on one GPU; the
    product's multi-GPU path is NCCL)."""
    import torch.distributed as dist

    return dist.get_backend(group) == "gloo"


def _all_reduce(t, group):
    import torch.distributed as dist

    if t.is_cuda and _staged(group):
        h = t.cpu()
        dist.all_reduce(h, group=group)
        t.copy_(h)
    else:
        dist.all_reduce(t, group=group)


def _all_gather(outs, t, group):
    import torch.distributed as dist

    if t.is_cuda and _staged(group):
        ho = [o.cpu() for o in outs]
        dist.all_gather(ho, t.cpu(), group=group)
        for o, h in zip(outs, ho):
            o.copy_(h)
    else:
        dist.all_gather(outs, t, group=group)


def _all_to_all(out, inp, group, out_splits=None, in_splits=None):
    import torch.distributed as dist

    if inp.is_cuda and _staged(group):
        ho = out.cpu()
        dist.all_to_all_single(ho, inp.cpu(), output_split_sizes=out_splits, input_split_sizes=in_splits,
                               group=group)
        out.copy_(ho)
    else:
        dist.all_to_all_single(out, inp, output_split_sizes=out_splits, input_split_sizes=in_splits, group=group)


def _targets(N: int, p: int):
    return [(t * N) // p for t in range(1, p)]


def exact_splitters(sorted_keys, n_local: int, group, ops, device):
    """Smallest v_t with global #(key <= v_t) >= k_t for t = 1..p-1, plus the
    per-rank send counts (rank-ordered tie split)."""
    import torch
    import torch.distributed as dist

    p = dist.get_world_size(group)
    r = dist.get_rank(group)
    nt = torch.tensor([n_local], dtype=torch.int64, device=device)
    _all_reduce(nt, group)
    N = int(nt.item())
    ks = _targets(N, p)
    lo = [0] * (p - 1)           # answer in [lo, hi]
    hi = [KEY_SPACE - 1] * (p - 1)
    rounds = 0
    while any(h > l for l, h in zip(lo, hi)):
        rounds += 1
        piv = []
        for t in range(p - 1):
            span = hi[t] - lo[t]
            m = PIVOTS_PER_TARGET
            # pivots lo + ceil(i * span / (m+1)) - 1 ... evenly splitting [lo, hi)
            cand = sorted({lo[t] + (i * span) // (m + 1) for i in range(1, m + 1)} - {hi[t]})
            cand = [c for c in cand if lo[t] <= c < hi[t]]
            cand = cand + [hi[t]] * (m - len(cand))
            piv.extend(cand)
        piv_np = np.array(piv, dtype=np.uint64).astype(np.uint32)
        _, le = ops.split_counts(sorted_keys, piv_np)
        le = le.to(torch.int64)
        _all_reduce(le, group)
        le_h = le.cpu().numpy()
        for t in range(p - 1):
            if hi[t] <= lo[t]:
                continue
            row = piv[t * PIVOTS_PER_TARGET:(t + 1) * PIVOTS_PER_TARGET]
            cnt = le_h[t * PIVOTS_PER_TARGET:(t + 1) * PIVOTS_PER_TARGET]
            new_lo, new_hi = lo[t], hi[t]
            for v, c in zip(row, cnt):       # row ascending
                if c >= ks[t]:
                    new_hi = min(new_hi, v)
                    break
                new_lo = max(new_lo, v + 1)
            lo[t], hi[t] = new_lo, new_hi
    vs = np.array(lo, dtype=np.uint64).astype(np.uint32)
    lt, le = ops.split_counts(sorted_keys, vs)
    lt = lt.to(torch.int64)
    eq = le.to(torch.int64) - lt
    both = torch.stack([lt, eq])                       # [2, p-1]
    gathered = [torch.empty_like(both) for _ in range(p)]
    _all_gather(gathered, both, group)
    G = torch.stack(gathered).cpu().numpy()            # [p, 2, p-1]
    cuts = [0]
    for t in range(p - 1):
        L = int(G[:, 0, t].sum())
        before = int(G[:r, 1, t].sum())
        take = min(int(G[r, 1, t]), max(0, ks[t] - L - before))
        cuts.append(int(G[r, 0, t]) + take)
    cuts.append(n_local)
    send = [cuts[d + 1] - cuts[d] for d in range(p)]
    return send, [int(v) for v in vs], rounds


class _PhaseMarks:
    """CUDA events on the current stream at the phase boundaries of one
    distributed sort (local_sort | splitters | exchange | merge); a no-op for
    non-CUDA tensors (gloo tests).  Read with phase_ms() after a synchronize."""

    NAMES = ("local_sort", "splitters", "exchange", "merge")

    def __init__(self, device, enabled: bool):
        import torch

        self.on = enabled and device.type == "cuda"
        self.ev = []
        self._torch = torch
        self.device = device

    def mark(self):
        if self.on:
            e = self._torch.cuda.Event(enable_timing=True)
            e.record(self._torch.cuda.current_stream(self.device))
            self.ev.append(e)

    def phase_ms(self) -> dict:
        if len(self.ev) != len(self.NAMES) + 1:
            return {}
        return {n: self.ev[i].elapsed_time(self.ev[i + 1]) for i, n in enumerate(self.NAMES)}


class _PeerMaps:
    """Peer allocations mapped into this process (CUDA IPC), by handle."""

    def __init__(self):
        self.maps = {}

    def base(self, bcf, handle: bytes) -> int:
        b = self.maps.get(handle)
        if b is None:
            b = bcf.ipc_open(handle)
            self.maps[handle] = b
        return b


_PEERS = _PeerMaps()


def _peer_exchange_merge(sk, send, group, ops, device):
    """Fused exchange + merge: every rank exports the IPC
    handle of its sorted shard, maps the others', and merges its p incoming
    runs -- slice [cut_s(r), cut_s(r+1)) of rank s's shard, read in place over
    NVLink -- with bcf_merge_runs_ptrs_u32, whose first pairwise pass reads the
    peers' memory directly: no receive buffer, no separate copy."""
    import torch
    import torch.distributed as dist

    bcf = ops.bcf
    p = dist.get_world_size(group)
    r = dist.get_rank(group)
    cuts = np.concatenate([[0], np.cumsum(send)]).astype(np.int64)
    handle, off = bcf.ipc_export(sk)
    info = [None] * p
    dist.all_gather_object(info, (handle, off, cuts.tolist()), group=group)
    # every shard complete before anyone reads it
    torch.cuda.current_stream(device).synchronize()
    dist.barrier(group)
    ptrs, lens = [], []
    for s_ in range(p):
        h, o, c = info[s_]
        base = sk.data_ptr() - off if s_ == r else _PEERS.base(bcf, h)
        ptrs.append(base + o + 4 * c[r])
        lens.append(c[r + 1] - c[r])
    out = bcf.merge_runs_ptrs(ptrs, lens, device, dtype=sk.dtype, params=ops.params)
    # the peers have read this rank's shard before it can be reused
    torch.cuda.current_stream(device).synchronize()
    dist.barrier(group)
    return out, lens


def sort(keys, values=None, group=None, ops=None, timing: list | None = None, exchange: str = "nccl"):
    """Distributed stable sort of the shards held by the ranks of `group`.
    Returns (keys_out, values_out_or_None, DistStats).  keys: 1-D 4-byte
    tensor (u32 bit patterns in int32); values likewise.  `timing`: if a
    list, a _PhaseMarks of this call is appended (CUDA tensors only).
    exchange: "nccl" (all_to_all_single, then bcf_merge_runs_u32) or "peer"
    (keys only, CUDA ops: the incoming runs are merged in place from the
    peers' memory over CUDA IPC / NVLink by bcf_merge_runs_ptrs_u32)."""
    import torch
    import torch.distributed as dist

    ops = ops or CudaOps()
    if getattr(keys, "dtype", None) is not None and str(keys.dtype) == "torch.float32":
        # the local sort orders float32 by IEEE totalOrder, but the splitters
        # and the run merge compare u32 bit patterns: pass keys as int32 bit
        # patterns (or totalOrder-encoded) instead of relying on a silent mismatch
        raise TypeError("dist.sort sorts 32-bit keys as unsigned bit patterns: pass int32 (uint32 bits), "
                        "not float32")
    device = keys.device
    p = dist.get_world_size(group)
    marks = _PhaseMarks(device, timing is not None and p > 1)
    marks.mark()
    sk, sv = ops.sort(keys, values)
    if p == 1:
        return sk, sv, DistStats(0, [keys.numel()], [keys.numel()], [])
    marks.mark()
    send, pivots, rounds = exact_splitters(sk, sk.numel(), group, ops, device)
    if exchange == "peer":
        if values is not None or not isinstance(ops, CudaOps) or device.type != "cuda":
            raise ValueError("exchange='peer' needs CUDA ops and keys only")
        marks.mark()
        ok, recv = _peer_exchange_merge(sk, send, group, ops, device)
        marks.mark()
        marks.mark()
        if timing is not None:
            timing.append(marks)
        return ok, None, DistStats(rounds, send, recv, pivots)
    elif exchange != "nccl":
        raise ValueError(f"unknown exchange {exchange!r}")
    sc = torch.tensor(send, dtype=torch.int64, device=device)
    rc = torch.empty_like(sc)
    _all_to_all(rc, sc, group)
    recv = [int(x) for x in rc.cpu().tolist()]
    marks.mark()
    rk = torch.empty(sum(recv), dtype=keys.dtype, device=device)
    _all_to_all(rk, sk, group, recv, send)
    rv = None
    if sv is not None:
        rv = torch.empty(sum(recv), dtype=values.dtype, device=device)
        _all_to_all(rv, sv, group, recv, send)
    marks.mark()
    offs = np.concatenate([[0], np.cumsum(recv)]).astype(np.uint64)
    ok, ov = ops.merge_runs(rk, offs, rv)
    marks.mark()
    if timing is not None:
        timing.append(marks)
    return ok, ov, DistStats(rounds, send, recv, pivots)
