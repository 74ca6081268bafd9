#!/bin/bash
# quick join check: the lane-join GPU parity tests + default bench
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_induced.py -x -q -k "c1 or c2_full or tiny or induced_c1 or ring" > gpurun_out/jq_test.log 2>&1; echo "pytest rc=$?" >> gpurun_out/jq_test.log
tail -2 gpurun_out/jq_test.log
for i in 1; do timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/jq_b.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/jq_b.json')); print(d['ms_per_step'], d['stage_ms'], d['find_first']['ms_per_step'])"; done
