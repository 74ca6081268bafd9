#!/bin/bash
# join A/B: default bench vs environment variants (VARIANTS="NAME=ENV ..."), FA + FF join times
mkdir -p gpurun_out
run() { env $2 timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ab_$1.json 2> gpurun_out/ab_$1.err;
  python -c "
import json; d=json.load(open('gpurun_out/ab_$1.json')); print('$1', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['stage_ms'].items()}, 'FF', round(d['find_first']['ms_per_step'],3))" || tail -3 gpurun_out/ab_$1.err; }
run base ""
for v in $VARIANTS; do run ${v%%=*} "${v#*=}"; done
