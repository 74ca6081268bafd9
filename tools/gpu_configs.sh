#!/bin/bash
# bench lines for configs[1], [3], [4] at two filter levels
mkdir -p gpurun_out
for L in 2 4; do
  for cfg in 1 3 4; do
    timeout 900 python bench.py --config $cfg --levels $L --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/cfg${cfg}_L$L.json 2> gpurun_out/cfg${cfg}_L$L.err
    python -c "
import json; d=json.load(open('gpurun_out/cfg${cfg}_L$L.json')); print('cfg $cfg L $L', round(d['ms_per_step'],3), '%.3e'%d['value'], d['unit'], d.get('stage_ms') or d.get('group_stage_ms'))" || tail -3 gpurun_out/cfg${cfg}_L$L.err
  done
done
