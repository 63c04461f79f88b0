#!/bin/bash
# One GPU session on the gpurun box: GPU tests, bench line, optional ncu.
#   tools/gpu_session.sh [tests] [bench] [ncu] [custom "cmd"]
# Outputs land in gpurun_out/ (merged back by gpurun).
set -u
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/gpu_info.txt 2>&1
for what in "$@"; do
  case "$what" in
    tests) timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" ;;
    bench) timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" ;;
    *) bash -c "$what"; echo "custom rc=$?" ;;
  esac
done
