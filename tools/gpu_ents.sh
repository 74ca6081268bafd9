#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
for e in 1 0; do
  SIGMO_JOIN_ENTS=$e timeout 600 python bench.py --no-cpu-baseline --steps 30 --warmup 5 --e2e-steps 1 > gpurun_out/sw.json 2> gpurun_out/sw.err
  python -c "
import json; d=json.load(open('gpurun_out/sw.json')); print('ents=$e', d['ms_per_step'], d['stage_ms'], d['find_first']['ms_per_step'])" || tail -3 gpurun_out/sw.err
done
