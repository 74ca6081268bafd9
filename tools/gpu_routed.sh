#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_stream.py -x -q > gpurun_out/pytest_stream.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_stream.log
tail -3 gpurun_out/pytest_stream.log
timeout 900 python bench.py --config 3 --steps 5 --warmup 3 > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err; tail -c 1500 gpurun_out/bench_cfg3.json; tail -3 gpurun_out/bench_cfg3.err
timeout 1200 python bench.py --config 4 --steps 2 --warmup 3 > gpurun_out/bench_cfg4.json 2> gpurun_out/bench_cfg4.err; tail -c 1500 gpurun_out/bench_cfg4.json; tail -3 gpurun_out/bench_cfg4.err
timeout 600 python bench.py --no-cpu-baseline --steps 30 --warmup 5 --e2e-steps 1 > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err
python -c "
import json; d=json.load(open('gpurun_out/bench_q.json')); print(d['ms_per_step'], d['value'], d['stage_ms'], d['find_first']['ms_per_step'])"
