#!/bin/bash
# configs[2] bench per library variant in build/variants/*.so (SIGMO_LIB)
mkdir -p gpurun_out
for v in ${@:-build/variants/*.so}; do
  SIGMO_LIB=$PWD/$v timeout 600 python bench.py --no-cpu-baseline --steps 30 --warmup 5 --e2e-steps 1 > gpurun_out/sw.json 2> gpurun_out/sw.err
  python -c "
import json; d=json.load(open('gpurun_out/sw.json')); print('$v', round(d['ms_per_step'],3), {k: round(x,3) for k,x in d['stage_ms'].items()}, round(d['find_first']['ms_per_step'],3))" || tail -3 gpurun_out/sw.err
done
