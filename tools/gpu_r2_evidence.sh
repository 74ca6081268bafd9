#!/bin/bash
# r2 evidence on the current tree: INT peak microbenchmark, ncu --set full of
# the bench's kernels (configs[2], L=2), ncu launch list of the bench command
mkdir -p gpurun_out
./tools/microbench/int_peak > gpurun_out/int_peak.json 2> gpurun_out/int_peak.err; cat gpurun_out/int_peak.json
L=${LEVELS:-2}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sigmo_filter_lane_jit|k_join_lane" -s 6 -c 3 -o gpurun_out/r2_full_L$L python tools/profile_step.py 1000000 $L 1 0 3 > gpurun_out/r2_full.log 2>&1
tail -1 gpurun_out/r2_full.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_ncu_bench.log 2>&1
tail -1 gpurun_out/r2_ncu_bench.log
