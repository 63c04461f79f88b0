#!/usr/bin/env python
"""bench.py -- headline benchmark of the B200 bank-conflict-free mergesort.

Metric (BASELINE.json): sorted keys/s (32-bit) on uniform-random vs constructed
worst-case inputs, their ratio, and (via ncu, profiles/) shared-memory bank
conflicts.  Workload at N = 1: BASELINE.json configs[1], 2^24 uint32 keys,
random vs worst-case, 1 x B200.  A step = one full sort (block sort + every
merge pass) of one batch of 2^24 keys already resident in HBM; timed steps
alternate random / worst-case (ABAB) so clock drift cancels in the ratio; L2
is flushed (256 MiB write) between timed steps, outside the events.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--log2n L]

N > 1 (torchrun, one rank per GPU, NCCL): BASELINE configs[4], 2^32 keys in
total (2^32 / N per rank, strong scaling), a step is the distributed sort
(local sort, exact splitters, all_to_all, run merge).  `--gpus 1 --log2n 32`
runs the same 2^32-key workload on one GPU.  Rank 0 prints ONE JSON line.
`--impl reference` times the CPU oracle (plain stable mergesort, 1 core) on
the same workload: the full input per step when the run fits a few minutes,
else a bounded sample (stated in cpu_baseline.sample).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synthetic_inputs as si  # noqa: E402

METRIC = "sorted keys/s (32-bit) random vs worst-case, ratio; SMEM bank conflicts (ncu)"
UNIT = "keys/s"
WORKLOAD_1 = "2^24 uint32 keys, random vs worst-case bank-conflict input, 1xB200 (BASELINE configs[1])"
WORKLOAD_DIST = "2^32 uint32 keys distributed sort (splitters + NCCL all-to-all over NVLink) (BASELINE configs[4])"
REF_BUDGET_S = 150.0  # the reference arm's whole run (warmup + steps) stays within a few minutes
L2_FLUSH_BYTES = 256 << 20
DEFAULT_E, DEFAULT_U = 31, 128  # = bcf_default_params()


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--log2n", type=int, default=0, help="total keys 2^L (default 24 at N=1, 32 at N>1)")
    ap.add_argument("--E", type=int, default=0)
    ap.add_argument("--u", type=int, default=0)
    ap.add_argument("--algo", type=int, default=0)
    ap.add_argument("--no-extras", action="store_true", help="skip e2e/cpu_baseline/contrast legs")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "peer"],
                    help="N > 1: all_to_all + run merge (nccl) or the fused peer-memory merge (peer)")
    return ap.parse_args()


def log2n_total(a, world):
    return a.log2n or (24 if world == 1 else 32)


def workload_config(a, world, E, u):
    """The `config` object, identical in both arms (ours / reference)."""
    L = log2n_total(a, world)
    n = 1 << L
    if L == 24 and world == 1:
        wl = WORKLOAD_1
    elif L == 32:
        wl = WORKLOAD_DIST if world > 1 else "2^32 uint32 keys, random vs worst-case, 1xB200 (BASELINE configs[4] at N=1)"
    else:
        wl = f"2^{L} uint32 keys, random vs worst-case, {world}xB200"
    return {"workload": wl, "n": n, "n_per_gpu": n // world, "E": E, "u": u,
            "algo": "conflict_free" if a.algo == 0 else "baseline",
            "steps_alternate": "random, worst-case (ABAB)",
            "l2": "flushed between timed steps (256 MiB write, outside the events)",
            "parallelism": f"dp{world}" if world > 1 else "single"}


def cpu_info():
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model,
            "affinity_cores": len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else None}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except OSError:
        return {"hbm_gbs": 6650.0}, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """NVML sampling of SM clock and throttle reasons during the timed region."""

    REASONS = [
        ("nvmlClocksEventReasonHwSlowdown", "hw_slowdown"),
        ("nvmlClocksEventReasonHwThermalSlowdown", "hw_thermal_slowdown"),
        ("nvmlClocksEventReasonSwThermalSlowdown", "sw_thermal_slowdown"),
        ("nvmlClocksEventReasonSwPowerCap", "sw_power_cap"),
        ("nvmlClocksEventReasonHwPowerBrakeSlowdown", "hw_power_brake_slowdown"),
        ("nvmlClocksEventReasonApplicationsClocksSetting", "applications_clocks_setting"),
        ("nvmlClocksEventReasonSyncBoost", "sync_boost"),
    ]

    def __init__(self, index: int):
        self.ok = False
        self.samples = []
        self.reasons = set()
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:  # noqa: BLE001
            self.max_mhz = None
        self._stop = threading.Event()

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for attr, name in self.REASONS:
                    if r & getattr(nv, attr, 0):
                        self.reasons.add(name)
            except Exception:  # noqa: BLE001
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def cpu_baselines(n: int, E: int, u: int, x_rand: np.ndarray, x_worst: np.ndarray):
    """(i) the oracle (plain stable mergesort in C, 1
    thread), (ii) std::stable_sort (1 thread), (iii) a std::thread parallel
    stable mergesort on all host cores; each on the same random and
    worst-case inputs as the GPU run (full size), outputs cross-checked."""
    import oracle

    info = cpu_info()
    cores = info["affinity_cores"] or info["nproc"] or 1
    res = {}
    exp = None
    for name, fn, c in [("oracle", oracle.sort_u32, 1), ("std_stable_sort", oracle.std_stable_sort_u32, 1),
                        ("parallel_mergesort", lambda x: oracle.parallel_mergesort_u32(x, cores), cores)]:
        secs = 0.0
        outs = []
        for x in (x_rand, x_worst):
            t = time.perf_counter()
            outs.append(fn(x))
            secs += time.perf_counter() - t
        if exp is None:
            exp = outs
        ok = all(np.array_equal(o, e) for o, e in zip(outs, exp))
        res[name] = {"value": 2 * n / secs, "unit": UNIT, "cores": c, "seconds": secs, "matches_oracle": ok}
    res["sample"] = f"one random + one worst-case sort of {n} keys each (the full workload)"
    res.update(info)
    return res


def extra_configs(bcf, dev, stream, flush, params, peaks, steps=10):
    """BASELINE configs[2]: 2^28 f32 keys and 2^26 u32 key-value pairs (stable),
    each timed like the headline (device-resident inputs, L2 flushed between
    steps, CUDA events on the launch stream), plus the merge pass's achieved
    HBM bandwidth (f32: 8 B/key, pairs: 16 B/pair per pass)."""
    import torch

    res = {}
    legs = [
        ("f32_2^28", 1 << 28, 8),
        ("pairs_u32_2^26", 1 << 26, 16),
        ("merge_u32_2x2^25", 1 << 26, 8),
        ("merge_runs_8x2^23", 1 << 26, 24),  # 3 pairwise passes x 8 B/key
        ("set_intersection_2x2^25", 1 << 26, 8),
    ]
    for name, n, bpk in legs:
        if name.startswith("f32"):
            x = si.uniform_f32_torch(n, si.config_seed(3), dev)
            out = torch.empty_like(x)
            run = lambda: bcf.sort(x, out=out, params=params, temp=temp)  # noqa: E731
            workload = "2^28 float32 keys, uniform [0,1) (24-bit mantissa grid), IEEE totalOrder"
        elif name.startswith("set_"):
            # bcf_set_op_u32: intersection of two sorted
            # 2^25 arrays drawn from 2^26 values (about half the keys common)
            prm = params
            sa_ = bcf.sort(si.uniform_u32_torch(n // 2, si.config_seed(7), dev) & 0x3FFFFFF, params=prm)
            sb_ = bcf.sort(si.uniform_u32_torch(n // 2, si.config_seed(7), dev, lo=n // 2) & 0x3FFFFFF, params=prm)
            run = lambda: bcf.set_op("intersection", sa_, sb_, params=prm)  # noqa: E731
            workload = ("bcf_set_op_u32 intersection of two sorted 2^25 uint32 arrays over 2^26 values "
                        "(tags, CF merge with tags, keep flags, compaction; includes the count read-back)")
        elif name.startswith("merge_runs"):
            # bcf_merge_runs_u32: the distributed sort's final local merge at p = 8
            prm = params
            rk = torch.cat([bcf.sort(si.uniform_u32_torch(n // 8, si.config_seed(6), dev, lo=r * (n // 8)),
                                     params=prm) for r in range(8)])
            roffs = np.arange(9, dtype=np.uint64) * np.uint64(n // 8)
            run = lambda: bcf.merge_runs(rk, roffs, params=prm)  # noqa: E731
            workload = "bcf_merge_runs_u32 of 8 sorted 2^23 uniform uint32 runs (3 CF merge passes)"
        elif name.startswith("merge"):
            # bcf_merge_u32: two separately allocated sorted halves
            prm = params
            ka = bcf.sort(si.uniform_u32_torch(n // 2, si.config_seed(5), dev), params=prm)
            kb = bcf.sort(si.uniform_u32_torch(n // 2, si.config_seed(5), dev, lo=n // 2), params=prm)
            mo = torch.empty(n, dtype=ka.dtype, device=dev)
            mtemp = bcf.merge_temp(n // 2, n // 2, params=prm, device=dev)
            run = lambda: bcf.merge(ka, kb, params=prm, out=mo, temp=mtemp)  # noqa: E731
            workload = ("bcf_merge_u32 of two sorted 2^25 uniform uint32 arrays (B reversed into temp, then one "
                        "pass of the window merge kernel)")
        else:
            k = si.dup_u32_torch(n, si.config_seed(4), dev)
            v = si.iota_u32_torch(n, dev)
            ko, vo = torch.empty_like(k), torch.empty_like(v)
            prm = bcf.default_pairs_params()  # pairs default (11, 256)
            run = lambda: bcf.sort_pairs(k, v, ko, vo, params=prm, temp=temp)  # noqa: E731
            workload = "2^26 uint32 (key & 0xFFFF, heavy duplicates) + uint32 value (index) pairs, stable"
        if name.startswith(("f32", "merge", "set_")):
            prm = params
        temp = bcf.temp_buffer(n, prm, pairs=name.startswith("pairs"), device=dev)
        for _ in range(3):
            run()
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
        for i in range(steps):
            flush.fill_(i)
            ev[i][0].record(stream)
            run()
            ev[i][1].record(stream)
        torch.cuda.synchronize()
        ms = sum(s.elapsed_time(e) for s, e in ev) / steps
        bcf.profile_enable(True)
        for i in range(3):
            flush.fill_(i)
            run()
        torch.cuda.synchronize()
        bcf.profile_enable(False)
        prof = bcf.profile_collect()
        cls = "merge_runs" if name.startswith("merge_runs") else ("merge" if name.startswith(("merge", "set_")) else
                                                                   ("merge_passes" if "merge_passes" in prof
                                                                    else "merge_pass"))
        mp = prof.get(cls, {"launches": 0, "total_ms": 0.0, "keys": 0})
        bs = prof.get("block_sort", {"launches": 0, "total_ms": 0.0})
        avg = mp["total_ms"] / max(1, mp["launches"])
        bpl = bpk * mp["keys"] / max(1, mp["launches"])  # keys counts n per pass
        res[name] = {"workload": workload, "n": n, "E": prm.items_per_thread, "u": prm.block_threads,
                     "value": n / (ms / 1e3),
                     "unit": "pairs/s" if name.startswith("pairs") else "keys/s", "ms_per_sort": ms,
                     "merge_pass": {"launches_per_sort": mp["launches"] // 3, "avg_ms": avg,
                                    "achieved_gbs": 8 * n / (avg / 1e3) / 1e9 if avg else None,
                                    "frac_of_hbm": (8 * n / (avg / 1e3) / 1e9) / peaks["hbm_gbs"] if avg else None,
                                    "bytes_per_launch": 8 * n} if name.startswith("merge_runs") else
                                   {"launches_per_sort": mp["launches"] // 3, "avg_ms": avg,
                                    "achieved_gbs": bpl / (avg / 1e3) / 1e9 if avg else None,
                                    "frac_of_hbm": (bpl / (avg / 1e3) / 1e9) / peaks["hbm_gbs"] if avg else None,
                                    "bytes_per_launch": bpl, "passes_per_launch": bpl / (bpk * n)},
                     # merge legs: algorithmic bytes of the whole call / call time
                     "call_gbs_algorithmic": bpk * n / (ms / 1e3) / 1e9 if name.startswith(("merge", "set_")) else None,
                     "block_sort_ms": bs["total_ms"] / max(1, bs["launches"])}
        del run, temp
        torch.cuda.empty_cache()
    return res


def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", str(a.gpus)))
    if rank != 0:
        return 0
    # the library's default (E, u) (tests/test_capi_host.py keeps these equal);
    # the reference arm runs no library code
    E, u = a.E or DEFAULT_E, a.u or DEFAULT_U
    n_full = 1 << log2n_total(a, world)
    import oracle
    from oracle import worstcase as wc

    # sample size: the full workload unless warmup + steps would exceed the
    # budget at the oracle's measured rate (~1 core, n log n)
    probe = si.uniform_u32(1 << 20, si.config_seed(1))
    t = time.perf_counter()
    oracle.sort_u32(probe)
    per_key = (time.perf_counter() - t) / (1 << 20) * (np.log2(n_full) / 20.0)
    budget_keys = int(REF_BUDGET_S / max(1, a.steps + a.warmup) / per_key)
    n_sample = n_full if budget_keys >= n_full else max(1 << 16, budget_keys)
    inputs = [si.uniform_u32(n_sample, si.config_seed(1)), wc.worst_case_input(n_sample, E, u, si.config_seed(1))]
    for i in range(a.warmup):
        oracle.sort_u32(inputs[i % 2])
    times = []
    for i in range(a.steps):
        t = time.perf_counter()
        oracle.sort_u32(inputs[i % 2])
        times.append(time.perf_counter() - t)
    total = sum(times)
    value = a.steps * n_sample / total
    rnd = [t for i, t in enumerate(times) if i % 2 == 0]
    wst = [t for i, t in enumerate(times) if i % 2 == 1]
    if n_sample == n_full:
        sample = f"the full workload: {n_sample} keys per step, random / worst-case alternating"
    else:
        sample = (f"{n_sample} keys per step (of the {n_full}-key workload, bounded to ~{REF_BUDGET_S:.0f} s), "
                  "random / worst-case alternating")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * total / a.steps,
        "higher_is_better": True, "scaling": "weak" if world == 1 else "strong", "vs_baseline": None,
        "dtype": "u32", "data": "synthetic", "config": workload_config(a, world, E, u),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                         **cpu_info()},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "random_keys_per_s": len(rnd) * n_sample / sum(rnd) if rnd else None,
        "worst_keys_per_s": len(wst) * n_sample / sum(wst) if wst else None,
        "worst_over_random_time": (statistics.mean(wst) / statistics.mean(rnd)) if rnd and wst else None,
    }
    print(json.dumps(line))
    return 0


def gen_uniform(n, seed, dev, lo=0, chunk=1 << 27):
    """Rank's shard [lo, lo + n) of the global uniform u32 stream, generated on
    the device in chunks (bounded temporaries at 2^32 keys)."""
    import torch

    t = torch.empty(n, dtype=torch.int32, device=dev)
    for c in range(0, n, chunk):
        m = min(chunk, n - c)
        t[c:c + m] = si.uniform_u32_torch(m, seed, dev, lo=lo + c)
    return t


def host_mem_available():
    try:
        import psutil

        return psutil.virtual_memory().available
    except Exception:  # noqa: BLE001
        return 0


def main():
    a = parse()
    if a.impl == "reference":
        return run_reference(a)
    import ctypes

    import torch
    import torch.distributed as dist

    import paper_conf_spaa_berneys25_b200 as bcf
    from paper_conf_spaa_berneys25_b200 import dist as bdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)

    dp = bcf.default_params()
    E = a.E or dp.items_per_thread
    u = a.u or dp.block_threads
    params = bcf.make_params(E, u, a.algo)
    L = log2n_total(a, world)
    n_total = 1 << L
    lo = (rank * n_total) // world
    n = ((rank + 1) * n_total) // world - lo
    seed = si.config_seed(1)
    config = workload_config(a, world, E, u)

    # inputs resident in HBM: rank r's shard of the global random stream, and
    # the Section-4 worst case for (E, u) built on the device
    x_rand = gen_uniform(n, seed, dev, lo=lo)
    x_worst = bcf.worst_case(n, E, u, seed + rank, device=dev)
    inputs = [x_rand, x_worst]
    out = torch.empty(n, dtype=torch.int32, device=dev)
    temp = bcf.temp_buffer(n, params, device=dev)
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.int32, device=dev)
    torch.cuda.synchronize()

    dist_marks, dist_sends = [], []

    def step(i, timing=None, x=None):
        x = inputs[i % 2] if x is None else x
        if world == 1:
            return bcf.sort(x, out=out, params=params, temp=temp)
        ko, _, st = bdist.sort(x, ops=bdist.CudaOps(params), timing=timing, exchange=a.exchange)
        if timing is not None:
            dist_sends.append(st.send_counts)
        return ko

    for i in range(max(3, a.warmup)):
        step(i)
    torch.cuda.synchronize()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = bcf.launch_count()
    with ClockSampler(local) as clk:
        for i in range(a.steps):
            flush.fill_(i)  # L2 flush, outside the events
            ev[i][0].record(stream)
            step(i)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
    launches = bcf.launch_count() - launches0
    if world > 1:
        dist.barrier()
    # Per-kernel durations (roofline): the library brackets each of its
    # launches with CUDA events on the launch stream.  Those event records sit
    # between kernels, so they are taken in a second, identical pass over the
    # same workload right after the headline region (which has none).
    bcf.profile_enable(True)
    for i in range(min(a.steps, 50 if L <= 28 else 6)):
        flush.fill_(i)
        step(i, timing=dist_marks if world > 1 else None)
    torch.cuda.synchronize()
    bcf.profile_enable(False)
    prof = bcf.profile_collect()
    distributed = None
    if world > 1 and dist_marks:
        # phase split of the distributed sort, from CUDA events
        # on the launch stream in the profiled pass; max over ranks.  Exchange
        # bandwidth = this rank's off-rank key bytes out / exchange time, against
        # NVLink 5's 900 GB/s per direction per GPU.
        names = list(bdist._PhaseMarks.NAMES)
        ph = [m.phase_ms() for m in dist_marks]
        mean_ms = [statistics.mean(p_[k] for p_ in ph) for k in names]
        offrank = statistics.mean(4 * (sum(sc) - sc[rank]) for sc in dist_sends)
        ex_rate = offrank / (mean_ms[names.index("exchange")] / 1e3) / 1e9
        tt = torch.tensor(mean_ms + [-ex_rate], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ph_max = tt.tolist()
        slowest = -ph_max[-1]  # min over ranks of the exchange rate
        distributed = {
            "phases_ms_max_over_ranks": dict(zip(names, ph_max[:-1])),
            "exchange": {"achieved_gbs_min_over_ranks": slowest, "peak": 900.0, "unit": "GB/s",
                         "frac": slowest / 900.0, "offrank_bytes_out_rank0": offrank,
                         "peak_source": "NVLink 5 per direction per GPU (nominal)"},
            "splitters": "exact, 64-ary bisection of the key space + rank-ordered tie split",
        }
    prof_ms = sum(v["total_ms"] for v in prof.values())
    ms = [s_.elapsed_time(e_) for s_, e_ in ev]
    # max over ranks of the timed region and of each half (random / worst)
    rnd_ms = sum(m for i, m in enumerate(ms) if i % 2 == 0)
    wst_ms = sum(m for i, m in enumerate(ms) if i % 2 == 1)
    t = torch.tensor([sum(ms), rnd_ms, wst_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_ms_max, rnd_ms, wst_ms = (float(v) for v in t.tolist())
    value = a.steps * n_total / (total_ms_max / 1e3)
    n_rnd = (a.steps + 1) // 2
    n_wst = a.steps // 2

    peaks, peak_src = measured_peaks()
    plan = bcf.sort_plan(n, params)
    T = plan["merge_tile"]
    passes = plan["merge_passes"]
    roof = None
    mcls = "merge_passes" if "merge_passes" in prof else "merge_pass"
    mp = prof.get(mcls)
    if mp and mp["launches"]:
        avg_ms = mp["total_ms"] / mp["launches"]
        # read 4 B + write 4 B per key per pass; "keys" counts n per pass
        # (a merge_passes launch runs every pass of one sort)
        bytes_per_launch = 8 * mp["keys"] / mp["launches"]
        achieved = bytes_per_launch / (avg_ms / 1e3) / 1e9
        traffic = None
        tf = os.path.join(ROOT, "profiles", "merge_pass_traffic.json")
        if os.path.exists(tf):
            with open(tf) as f:
                tr = json.load(f)
            if tr.get("n") == n and tr.get("E") == E and tr.get("u") == u:
                traffic = tr.get("dram_bytes_per_launch")
        bs = prof.get("block_sort")
        in_region = None
        if bs and bs["launches"] and passes and world == 1:
            # the profiled pass brackets every launch with events, which
            # serialises the launches (no PDL overlap); the headline region has
            # none: its merge time per launch, net of the event-timed block sort
            in_region = (total_ms_max / a.steps - bs["total_ms"] / bs["launches"]) / (
                passes if mcls == "merge_pass" else 1)
        roof = {"bound": "hbm", "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": achieved / peaks["hbm_gbs"], "traffic": traffic,
                "kernel": mcls, "avg_launch_ms": avg_ms, "bytes_per_launch": bytes_per_launch,
                "passes_per_launch": passes if mcls == "merge_passes" else 1,
                "merge_pass_in_region_est_ms": in_region,
                "achieved_in_region_est": (bytes_per_launch / (in_region / 1e3) / 1e9) if in_region else None,
                "peak_source": f"hbm_gbs {peak_src} (MEASURED_PEAKS.json copy bandwidth)"}
    kernels = {k: {"launches": v["launches"], "avg_ms": v["total_ms"] / max(1, v["launches"]),
                   "share_of_kernel_time": v["total_ms"] / prof_ms if prof_ms else None}
               for k, v in prof.items()}

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
        "warmup": max(3, a.warmup), "ms_per_step": total_ms_max / a.steps, "higher_is_better": True,
        "scaling": "weak" if world == 1 else "strong", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic", "config": config,
        "plan": {"tile": T, "block_sort_tile": plan["block_sort_tile"], "merge_passes": passes},
        "roofline": roof,
        "kernels": kernels,
        "gpu_launches": launches,
        "clocks": clk.summary(),
    }
    if distributed is not None:
        distributed["exchange_mode"] = a.exchange
        if a.exchange == "nccl":
            # context: the fused exchange + merge over peer memory on
            # the same inputs, timed the same way (max over ranks)
            try:
                kp = min(a.steps, 10)
                for i in range(2):
                    bdist.sort(inputs[i % 2], ops=bdist.CudaOps(params), exchange="peer")
                pev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(kp)]
                dist.barrier()
                torch.cuda.synchronize()
                for i in range(kp):
                    flush.fill_(i)
                    pev[i][0].record(stream)
                    bdist.sort(inputs[i % 2], ops=bdist.CudaOps(params), exchange="peer")
                    pev[i][1].record(stream)
                torch.cuda.synchronize()
                pt = torch.tensor([sum(s_.elapsed_time(e_) for s_, e_ in pev)], dtype=torch.float64, device=dev)
                dist.all_reduce(pt, op=dist.ReduceOp.MAX)
                distributed["peer_exchange_keys_per_s"] = kp * n_total / (float(pt.item()) / 1e3)
            except Exception as ex:  # noqa: BLE001
                distributed["peer_exchange_error"] = repr(ex)[:200]
        line["distributed"] = distributed

    # ---- e2e through the public API, host buffers, copies inside the region
    big = n > (1 << 28)
    if not a.no_extras or world > 1 or big:
        need = 4 * 4 * n if (world == 1 and not big) else 2 * 4 * n
        if host_mem_available() > 2 * need * (world if world > 1 else 1):
            line["e2e"] = e2e_leg(a, bcf, bdist, torch, dist, dev, stream, inputs, out, temp, params, n,
                                  n_total, world, big)
        else:
            line["e2e"] = {"value": None, "unit": UNIT, "skipped": "not enough host memory for pinned buffers",
                           "h2d_bytes_per_step": 4 * n, "d2h_bytes_per_step": 4 * n}

    if rank == 0 and world == 1 and not a.no_extras and not big:
        line["contrast"] = contrast_leg(bcf, torch, dev, stream, flush, x_rand, out, n, u, seed, a.steps)
        line["configs_extra"] = extra_configs(bcf, dev, stream, flush, params, peaks)
        xr = x_rand.cpu().numpy().view(np.uint32)
        xw = x_worst.cpu().numpy().view(np.uint32)
        cb = cpu_baselines(n, E, u, xr, xw)
        orc = cb.pop("oracle")
        line["cpu_baseline"] = {"value": orc["value"], "unit": UNIT, "cores": 1, "kind": "oracle",
                                "sample": cb.pop("sample"), **cb}
    # the headline ratio last, so it survives any tail truncation of stdout
    line["random_keys_per_s"] = n_rnd * n_total / (rnd_ms / 1e3) if n_rnd else None
    line["worst_keys_per_s"] = n_wst * n_total / (wst_ms / 1e3) if n_wst else None
    line["worst_over_random_time"] = ((wst_ms / n_wst) / (rnd_ms / n_rnd)) if n_rnd and n_wst else None
    if rank == 0:
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()
    return 0


def e2e_leg(a, bcf, bdist, torch, dist, dev, stream, inputs, out, temp, params, n, n_total, world, big):
    """The metric end to end through the public API: every step copies that
    step's input from pinned host memory to the device, sorts it, and reads
    the sorted keys back; the copies are inside the timed region."""
    hx = [x.cpu().pin_memory() for x in inputs]
    if world == 1 and not big:
        # bcf_sort_u32_host_batch: H2D / sort / D2H of consecutive steps overlap
        hy = [torch.empty(n, dtype=torch.int32).pin_memory() for _ in range(2)]
        ke = min(a.steps, 40)
        h_in = [hx[i % 2] for i in range(ke)]
        h_out = [hy[i % 2] for i in range(ke)]
        bcf.sort_host_batch(h_in[:4], h_out[:4], params=params, device=dev)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        bcf.sort_host_batch(h_in, h_out, params=params, device=dev)
        e1.record(stream)
        torch.cuda.synchronize()
        return {"value": ke * n / (e0.elapsed_time(e1) / 1e3), "unit": UNIT, "h2d_bytes_per_step": 4 * n,
                "d2h_bytes_per_step": 4 * n, "steps": ke,
                "api": "bcf_sort_u32_host_batch (pinned host buffers, H2D/sort/D2H of consecutive steps overlap)"}
    # one step per call: H2D, sort (distributed at N > 1), D2H; max over ranks
    hy = torch.empty(n, dtype=torch.int32).pin_memory()
    dx = torch.empty(n, dtype=torch.int32, device=dev)
    ke = 4
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(ke)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for i in range(ke):
        evs[i][0].record(stream)
        dx.copy_(hx[i % 2], non_blocking=True)
        if world == 1:
            r = bcf.sort(dx, out=out, params=params, temp=temp)
        else:
            r, _, _ = bdist.sort(dx, ops=bdist.CudaOps(params))
        hr = hy[:r.numel()]
        hr.copy_(r, non_blocking=True)
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    tot = torch.tensor([sum(s_.elapsed_time(e_) for s_, e_ in evs)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    return {"value": ke * n_total / (float(tot.item()) / 1e3), "unit": UNIT, "h2d_bytes_per_step": 4 * n,
            "d2h_bytes_per_step": 4 * n, "steps": ke,
            "api": ("dist.sort (one step per call: H2D of the rank's shard, distributed sort, D2H of the "
                    "rank's output), max over ranks") if world > 1 else
                   "bcf.sort (one step per call: H2D, sort, D2H; no overlap)"}


def contrast_leg(bcf, torch, dev, stream, flush, x_rand, out, n, u, seed, steps):
    """The unmodified-Thrust baseline variant (BCF_ALGO_BASELINE) on the same
    random input and on the Section-4 worst case built for ITS (E, u), beside
    the CF kernels with the same (E, u): E = 31 (our default) and E = 15 (the
    paper's)."""
    contrast = {}
    for E_ in (31, 15):
        for name, algo in (("baseline_thrust", bcf.ALGO_BASELINE), ("cf", 0)):
            prm = bcf.make_params(E_, u, algo)
            xw = bcf.worst_case(n, E_, u, seed, device=dev)
            ins = [x_rand, xw]
            tmp2 = bcf.temp_buffer(n, prm, device=dev)
            for i in range(4):
                bcf.sort(ins[i % 2], out=out, params=prm, temp=tmp2)
            kc = min(steps, 60)
            cev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(kc)]
            for i in range(kc):
                flush.fill_(i)
                cev[i][0].record(stream)
                bcf.sort(ins[i % 2], out=out, params=prm, temp=tmp2)
                cev[i][1].record(stream)
            torch.cuda.synchronize()
            cm = [s.elapsed_time(e) for s, e in cev]
            r_ = [m for i, m in enumerate(cm) if i % 2 == 0]
            w_ = [m for i, m in enumerate(cm) if i % 2 == 1]
            contrast[f"{name}_E{E_}"] = {"E": E_, "u": u,
                                         "random_keys_per_s": len(r_) * n / (sum(r_) / 1e3),
                                         "worst_keys_per_s": len(w_) * n / (sum(w_) / 1e3),
                                         "worst_over_random_time": statistics.mean(w_) / statistics.mean(r_)}
            del xw, tmp2
    return contrast


if __name__ == "__main__":
    sys.exit(main())
