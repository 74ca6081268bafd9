#!/bin/bash
mkdir -p gpurun_out
for T in 1 2 3 4; do
  SIGMO_TAIL_MAX=$T timeout 600 python bench.py --no-cpu-baseline --steps 20 --warmup 3 --e2e-steps 1 > gpurun_out/bench_t$T.json 2> gpurun_out/bench_t$T.err
  python -c "
import json; d=json.load(open('gpurun_out/bench_t$T.json')); print('tail', $T, d['ms_per_step'], d['stage_ms'], d['find_first']['ms_per_step'], d['roofline_join']['dfs_steps_per_launch'], d['counts']['matches'])"
done
