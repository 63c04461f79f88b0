#!/usr/bin/env python
"""Run a fixed list of sorts for an ncu bank-conflict capture.

Each configuration (algo, E, u, input kind, n) is sorted once after a warm-up
call; the script prints, to stderr, the launch index range each configuration
occupies so the ncu CSV (one row per launch and metric) can be attributed.
Usage under ncu:
  ncu --metrics <bank-conflict metrics> --csv --log-file gpurun_out/conf.csv \
      python tools/conflicts.py --n 16777216 --configs cf:16:256,base:15:256,...
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402
import synthetic_inputs as si  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 24)
    ap.add_argument("--configs", default="cf:16:256,cf:15:256,base:15:256,cf:17:256,base:17:256")
    ap.add_argument("--kinds", default="random,worst")
    ap.add_argument("--out", default="gpurun_out/conflicts_map.json")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    n = a.n
    x_rand = si.uniform_u32_torch(n, si.config_seed(1), dev)
    mapping = []
    seen = 0  # library launches of the sorts so far (the ncu -k filter drops the generator's)
    for cfg in a.configs.split(","):
        algo, E, u = cfg.split(":")
        E, u = int(E), int(u)
        prm = bcf.make_params(E, u, bcf.ALGO_BASELINE if algo == "base" else bcf.ALGO_CONFLICT_FREE)
        for kind in a.kinds.split(","):
            x = x_rand if kind == "random" else bcf.worst_case(n, E, u, si.config_seed(1), device=dev)
            torch.cuda.synchronize()
            first = bcf.launch_count()
            bcf.sort(x, params=prm)
            torch.cuda.synchronize()
            last = bcf.launch_count()
            mapping.append({"algo": algo, "E": E, "u": u, "kind": kind, "n": n,
                            "first_launch": seen, "launches": last - first})
            seen += last - first
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(mapping, f, indent=1)
    print(json.dumps(mapping), file=sys.stderr)


if __name__ == "__main__":
    main()
