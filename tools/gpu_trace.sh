# timeline of one merge pass (BCF_TRACE) + source-level ncu capture of the merge pass
mkdir -p gpurun_out
BCF_TRACE=6 timeout 300 python tools/trace_pass.py > gpurun_out/trace_p6.txt 2>&1
BCF_TRACE=12 timeout 300 python tools/trace_pass.py > gpurun_out/trace_p12.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:merge_pass -s 20 -c 1 -o gpurun_out/prof_merge -f python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/prof_merge.log 2>&1
echo done
