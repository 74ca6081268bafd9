#!/bin/bash
mkdir -p gpurun_out
for b in 2 4 8 16; do
  SIGMO_JOIN_BATCH=$b timeout 600 python bench.py --no-cpu-baseline --steps 20 --warmup 3 --e2e-steps 1 > gpurun_out/sw.json 2> gpurun_out/sw.err
  python -c "
import json; d=json.load(open('gpurun_out/sw.json')); print('batch=$b', d['stage_ms']['join'], d['find_first']['ms_per_step'])" || tail -3 gpurun_out/sw.err
done
