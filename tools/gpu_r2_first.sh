#!/bin/bash
# r2 first GPU call: GPU test suite on the r1 tree, compute-sanitizer
# memcheck / racecheck / synccheck over tools/sanitize_cases.py, default bench
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2_smi.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2_gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r2_gputest.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_cases.py > gpurun_out/r2_sanitizer_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/r2_sanitizer_$tool.log
done
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/r2_bench0.json 2> gpurun_out/r2_bench0.err
tail -3 gpurun_out/r2_gputest.log
for tool in memcheck racecheck synccheck; do tail -3 gpurun_out/r2_sanitizer_$tool.log; done
