#!/bin/bash
# join blocks-per-SM sweep on configs[2]
mkdir -p gpurun_out
for B in ${@:-4 5 6 8}; do
  SIGMO_JOIN_BPS=$B timeout 120 python bench.py --no-cpu-baseline --steps 20 --warmup 3 --e2e-steps 1 > gpurun_out/bench_b$B.json 2> gpurun_out/bench_b$B.err
  python -c "
import json; d=json.load(open('gpurun_out/bench_b$B.json')); print('bps', $B, round(d['ms_per_step'],3), {k:round(v,3) for k,v in d['stage_ms'].items()}, 'FF', round(d['find_first']['ms_per_step'],3))" || tail -3 gpurun_out/bench_b$B.err
done
