#!/bin/bash
# ncu --set full capture of the top kernels at configs[2] (1M molecules); summaries under gpurun_out/
mkdir -p gpurun_out
N=${1:-1000000}
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_join_lane|k_filter|k_pairs" -c 4 \
  -o gpurun_out/full_c2 -f python tools/profile_step.py $N 4 1 0 3 > gpurun_out/ncu_full.log 2>&1
python tools/ncu_summary.py gpurun_out/full_c2.ncu-rep > gpurun_out/full_c2_summary.md 2>&1
true
