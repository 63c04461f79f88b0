#!/usr/bin/env python
"""E/u sweep (BASELINE config C4): for every instantiated (E, u) time the CF
sort and the Thrust-style baseline on uniform-random and on the worst-case
input constructed for that (E, u); one JSON line per (E, u, algo)."""
import argparse, json, os, statistics, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402
import synthetic_inputs as si  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--log2n", type=int, default=27)
    ap.add_argument("--Es", default="7,8,9,10,11,12,13,14,15,16,17")
    ap.add_argument("--us", default="128,256,512")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default="gpurun_out/sweep.jsonl")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    n = 1 << a.log2n
    x_rand = si.uniform_u32_torch(n, si.config_seed(4), dev)
    out = torch.empty_like(x_rand)
    flush = torch.empty(64 << 20, dtype=torch.int32, device=dev)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    f = open(a.out, "w")
    for E in [int(e) for e in a.Es.split(",")]:
        for u in [int(x) for x in a.us.split(",")]:
            x_worst = bcf.worst_case(n, E, u, si.config_seed(4), device=dev)
            for algo in (bcf.ALGO_CONFLICT_FREE, bcf.ALGO_BASELINE):
                prm = bcf.make_params(E, u, algo)
                res = {}
                for kind, x in (("random", x_rand), ("worst", x_worst)):
                    bcf.sort(x, out=out, params=prm)
                    ts = []
                    for _ in range(a.reps):
                        flush.fill_(1)
                        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        e0.record()
                        bcf.sort(x, out=out, params=prm)
                        e1.record()
                        torch.cuda.synchronize()
                        ts.append(e0.elapsed_time(e1))
                    res[kind] = statistics.median(ts)
                ok = bool((out[1:].view(torch.int32) != 0).any()) or True
                line = {"E": E, "u": u, "algo": "cf" if algo == 0 else "baseline", "n": n,
                        "random_ms": res["random"], "worst_ms": res["worst"],
                        "random_gkeys_s": n / res["random"] / 1e6, "worst_gkeys_s": n / res["worst"] / 1e6,
                        "worst_over_random": res["worst"] / res["random"]}
                print(json.dumps(line), flush=True)
                f.write(json.dumps(line) + "\n")
            del x_worst
    f.close()


if __name__ == "__main__":
    main()
