#!/bin/bash
# sweep the JIT filter's min-CTAs-per-SM bound (register cap) at configs[2]
mkdir -p gpurun_out
for mb in 2 3 4 5; do
  SIGMO_FILTER_JIT_MINB=$mb timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/minb_$mb.json 2> gpurun_out/minb_$mb.err
  python -c "
import json; d=json.load(open('gpurun_out/minb_$mb.json')); print('minb $mb', d['ms_per_step'], d['stage_ms'])"
done
