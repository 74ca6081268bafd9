#!/bin/bash
# join occupancy / carve-out sweep at configs[2]
mkdir -p gpurun_out
for cfg in "9 -1" "6 -1" "6 50" "4 -1" "4 30" "9 75"; do
  set -- $cfg
  if [ "$2" = "-1" ]; then unset SIGMO_JOIN_CARVE; else export SIGMO_JOIN_CARVE=$2; fi
  SIGMO_JOIN_BPS=$1 timeout 600 python bench.py --no-cpu-baseline --steps 20 --warmup 3 --e2e-steps 1 > gpurun_out/sw.json 2> gpurun_out/sw.err
  python -c "
import json; d=json.load(open('gpurun_out/sw.json')); print('bps=$1 carve=$2', d['stage_ms']['join'], d['find_first']['ms_per_step'])" || tail -3 gpurun_out/sw.err
done
