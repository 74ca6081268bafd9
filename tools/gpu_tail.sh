#!/bin/bash
# parity tests (default planner) + configs[2] bench per SIGMO_TAIL_MAX
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/pytest_gpu.log
for t in 1 2 3 4; do
  SIGMO_TAIL_MAX=$t timeout 600 python bench.py --no-cpu-baseline --steps 30 --warmup 5 --e2e-steps 1 > gpurun_out/bench_tail$t.json 2> gpurun_out/bench_tail$t.err
  python -c "
import json; d=json.load(open('gpurun_out/bench_tail$t.json')); print('tail$t', d['ms_per_step'], '%.4g'%d['value'], d['stage_ms'], d['find_first']['ms_per_step'], d['counts']['matches'], d['roofline_join']['dfs_steps_per_launch'])"
done
