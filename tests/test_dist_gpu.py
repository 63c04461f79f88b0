"""The distributed sort (paper_conf_spaa_berneys25_b200/dist.py) with the REAL
CUDA ops (local CF sort, device split counts, CF run merge through the C ABI)
at world size 2 on the one GPU of the test box: two processes share cuda:0,
collectives run over gloo on host-staged copies.  Rank r's output must equal
positions [floor(rN/p), floor((r+1)N/p)) of the oracle's stable sort of the
concatenated global input."""
import os
import socket

import numpy as np
import pytest

import oracle
import synthetic_inputs as si

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _global_input(case):
    n_total, mask, _ = case
    return si.uniform_u32(n_total, 4321) & np.uint32(mask), si.iota_u32(n_total)


def _worker(rank, world, port, case, q, exchange="nccl"):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import paper_conf_spaa_berneys25_b200 as bcf
    from paper_conf_spaa_berneys25_b200 import dist as bdist

    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        dev = torch.device("cuda", 0)
        n_total, _, with_vals = case
        lo, hi = (rank * n_total) // world, ((rank + 1) * n_total) // world
        gk, gv = _global_input(case)
        kt = torch.from_numpy(gk[lo:hi].view(np.int32).copy()).to(dev)
        vt = torch.from_numpy(gv[lo:hi].view(np.int32).copy()).to(dev) if with_vals else None
        launches0 = bcf.launch_count()
        ok, ov, st = bdist.sort(kt, vt, ops=bdist.CudaOps(), exchange=exchange)
        torch.cuda.synchronize()
        assert ok.is_cuda and bcf.launch_count() > launches0   # the library ran
        q.put((rank, ok.cpu().numpy().view(np.uint32).copy(),
               None if ov is None else ov.cpu().numpy().view(np.uint32).copy(), st.send_counts))
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e), None, None))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case,exchange", [
    ((300001, 0xFFFFFFFF, True), "nccl"),    # distinct-ish keys, pairs, many tiles per rank
    ((200000, 0x7, True), "nccl"),           # 8 distinct keys: ties across the cut, stability
    ((123457, 0xFFFFFFFF, False), "nccl"),   # keys only, ragged
    ((123457, 0xFFFFFFFF, False), "peer"),   # fused exchange + merge over CUDA IPC (f1)
    ((400000, 0x3, False), "peer"),          # 4 distinct keys: ties across ranks, run order
    ((3, 0xFF, False), "peer"),              # tiny: empty incoming runs
])
def test_dist_sort_cuda_ops_world2_one_gpu(case, exchange):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q, exchange)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        r, k, v, sc = q.get(timeout=600)
        assert not isinstance(k, str), k
        res[r] = (k, v)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    gk, gv = _global_input(case)
    ek, ev = oracle.sort_pairs_u32(gk, gv)
    for r in range(world):
        k, v = res[r]
        np.testing.assert_array_equal(k, oracle.dist_rank_slice(ek, r, world))
        if case[2]:
            np.testing.assert_array_equal(v, oracle.dist_rank_slice(ev, r, world))
