#!/bin/bash
# r1 evidence refresh after the induced-mode changes: smoke, default bench (configs[2] + cpu_baseline),
# reference arm, ncu launch list of the default bench command
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_bench.log 2>&1
tail -2 gpurun_out/smoke.log
python -c "
import json; d=json.load(open('gpurun_out/bench_c2.json')); print(d['ms_per_step'], d['value'], d['stage_ms'], d['cpu_baseline']['value'], d['clocks'])"
