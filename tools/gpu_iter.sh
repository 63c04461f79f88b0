# iteration: GPU parity (fail fast) + bench lines at 2^24 / 2^27 + timeline of one pass
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x --timeout 300 --tb=short > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
for ln in 24 27; do
  timeout 300 python bench.py --log2n $ln --steps 40 --no-extras 2>/dev/null | tail -1 > gpurun_out/bench_$ln.json
done
BCF_TRACE=6 timeout 300 python tools/trace_pass.py > gpurun_out/trace_p6.txt 2>&1
echo done
