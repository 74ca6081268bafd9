#!/bin/bash
# r2 iteration: GPU parity suite, default bench, ncu of the filter, sanitizer (lane case)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/it_gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/it_gputest.log
SIGMO_DEBUG_FILTER=1 timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/it_bench.json 2> gpurun_out/it_bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${NCU_K:-sigmo_filter_lane_jit} -s 2 -c 1 -o gpurun_out/${NCU_NAME:-filt} python tools/profile_step.py 1000000 4 1 0 3 > gpurun_out/ncu_lane.log 2>&1
if [ -n "$SANITIZE" ]; then
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_cases.py > gpurun_out/r2_sanitizer_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/r2_sanitizer_$tool.log
  tail -2 gpurun_out/r2_sanitizer_$tool.log
done
fi
tail -4 gpurun_out/it_gputest.log
python -c "
import json; d=json.load(open('gpurun_out/it_bench.json')); print(d['ms_per_step'], d['value'], d['stage_ms'], d['clocks'], d['find_first'])" || tail -20 gpurun_out/it_bench.err
tail -2 gpurun_out/ncu_lane.log
