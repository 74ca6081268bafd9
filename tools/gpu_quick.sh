#!/bin/bash
# quick GPU iteration: gpu tests + configs[2] bench (no cpu baseline)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -30 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline --steps 50 --warmup 5 --e2e-steps 1 > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err
python -c "
import json; d=json.load(open('gpurun_out/bench_q.json')); print(d['ms_per_step'], d['value'], d['stage_ms'], d['find_first']['ms_per_step'], d['roofline_join']['dfs_steps_per_launch'])" 
tail -3 gpurun_out/bench_q.err
