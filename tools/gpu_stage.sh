#!/bin/bash
mkdir -p gpurun_out
SIGMO_JOIN_STAGE=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c2_full or c3_bench or random_tiny or fig3 or edge or c1_bitmap" > gpurun_out/pytest_stage.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_stage.log
tail -3 gpurun_out/pytest_stage.log
for st in 0 1; do
  SIGMO_JOIN_STAGE=$st timeout 600 python bench.py --no-cpu-baseline --steps 30 --warmup 5 --e2e-steps 1 > gpurun_out/sw.json 2> gpurun_out/sw.err
  python -c "
import json; d=json.load(open('gpurun_out/sw.json')); print('stage=$st', round(d['ms_per_step'],3), {k: round(x,3) for k,x in d['stage_ms'].items()}, round(d['find_first']['ms_per_step'],3))" || tail -3 gpurun_out/sw.err
done
