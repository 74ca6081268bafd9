#!/bin/bash
# join iteration: GPU parity (without the full-size file unless FULL=1), default bench, ncu of the lane join
mkdir -p gpurun_out
K=${PYTEST_K:-"not fullsize"}
[ -n "$FULL" ] && K=""
timeout 1500 python -m pytest tests -m gpu -x -q ${K:+-k "$K"} > gpurun_out/it_gputest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/it_gputest.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 1 > gpurun_out/it_bench.json 2> gpurun_out/it_bench.err
[ -n "$INDUCED" ] && timeout 600 python bench.py --induced --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/it_bench_ind.json 2> gpurun_out/it_bench_ind.err
if [ -z "$NO_NCU" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_join_lane -s ${NCU_S:-2} -c 2 -o gpurun_out/${NCU_NAME:-join_it} python tools/profile_step.py 1000000 2 1 0 3 > gpurun_out/ncu_join_it.log 2>&1
fi
tail -4 gpurun_out/it_gputest.log
for f in gpurun_out/it_bench.json gpurun_out/it_bench_ind.json; do [ -f $f ] && python -c "
import json; d=json.load(open('$f')); print(d['ms_per_step'], d['value'], d['stage_ms'], d['clocks'], d['find_first'], d['roofline'].get('dfs_steps_per_launch'))"; done
tail -20 gpurun_out/it_bench.err | grep -v "^$" | tail -5
tail -2 gpurun_out/ncu_join_it.log
