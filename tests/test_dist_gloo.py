"""Host logic of the distributed sort (paper_conf_spaa_berneys25_b200/dist.py)
on CPU with the gloo backend, world size 2 and 4: exact splitters, rank-ordered
tie split, all_to_all exchange, run-order merge.  The local GPU phases are
replaced by numpy test doubles (injected `ops`); the expected result is the
oracle's stable sort of the concatenated global input, sliced per rank."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synthetic_inputs as si
from paper_conf_spaa_berneys25_b200 import dist as bdist


class NumpyOps:
    """Test double for the three local phases (CPU tensors)."""

    def sort(self, keys, values=None):
        k = keys.numpy().view(np.uint32)
        perm = np.argsort(k, kind="stable")
        ks = torch.from_numpy(k[perm].view(np.int32).copy())
        if values is None:
            return ks, None
        return ks, torch.from_numpy(values.numpy()[perm].copy())

    def split_counts(self, sorted_keys, pivots_u32):
        k = sorted_keys.numpy().view(np.uint32)
        lt = np.searchsorted(k, pivots_u32.astype(np.uint32), side="left").astype(np.int64)
        le = np.searchsorted(k, pivots_u32.astype(np.uint32), side="right").astype(np.int64)
        return torch.from_numpy(lt), torch.from_numpy(le)

    def merge_runs(self, keys, offsets, values=None):
        return self.sort(keys, values)  # stable sort of the run-ordered concatenation


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n_total, mask, with_vals, skew = case
        lo = (rank * n_total) // world
        hi = ((rank + 1) * n_total) // world
        if skew:  # unequal shard sizes
            lo = [0, 3, n_total // 2, n_total - 5, n_total][rank] if world == 4 else [0, 7, n_total][rank]
            hi = [3, n_total // 2, n_total - 5, n_total, n_total][rank] if world == 4 else [7, n_total][rank]
        keys = si.uniform_u32(hi - lo, 1234, lo=lo) & np.uint32(mask)
        vals = si.iota_u32(hi - lo, lo=lo)
        kt = torch.from_numpy(keys.view(np.int32).copy())
        vt = torch.from_numpy(vals.view(np.int32).copy()) if with_vals else None
        tm = []
        ok, ov, st = bdist.sort(kt, vt, ops=NumpyOps(), timing=tm)
        assert len(tm) == 1 and tm[0].phase_ms() == {}  # phase events are CUDA-only
        q.put((rank, ok.numpy().view(np.uint32).copy(),
               None if ov is None else ov.numpy().view(np.uint32).copy(), st.rounds))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("case", [
    (10000, 0xFFFFFFFF, True, False),   # distinct-ish keys
    (10000, 0x3, True, False),          # 4 distinct keys: ties across ranks
    (5001, 0x0, True, False),           # all keys equal
    (777, 0xFF, False, True),           # unequal shard sizes, keys only
])
def test_dist_sort_matches_oracle_slices(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        r, k, v, rounds = q.get(timeout=120)
        res[r] = (k, v, rounds)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    n_total, mask, with_vals, _ = case
    gk = si.uniform_u32(n_total, 1234) & np.uint32(mask)
    gv = si.iota_u32(n_total)
    ek, ev = oracle.sort_pairs_u32(gk, gv)
    for r in range(world):
        k, v, rounds = res[r]
        np.testing.assert_array_equal(k, oracle.dist_rank_slice(ek, r, world))
        if with_vals:
            np.testing.assert_array_equal(v, oracle.dist_rank_slice(ev, r, world))
        assert rounds <= 7
