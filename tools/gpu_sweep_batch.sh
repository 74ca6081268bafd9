#!/bin/bash
mkdir -p gpurun_out
for b in ${@:-6 8 12 16 24}; do
  SIGMO_JOIN_BATCH=$b timeout 600 python bench.py --no-cpu-baseline --steps 20 --warmup 3 --e2e-steps 1 > gpurun_out/sw.json 2> gpurun_out/sw.err
  python -c "
import json; d=json.load(open('gpurun_out/sw.json')); print('batch=$b', round(d['stage_ms']['join'],3), round(d['find_first']['ms_per_step'],3))" || tail -3 gpurun_out/sw.err
done
