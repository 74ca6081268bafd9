#!/bin/bash
# ncu --set full of the join (and filter) at configs[2] with N molecules
mkdir -p gpurun_out
N=${1:-200000}
TAG=${2:-join}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_join_lane" -c 1 \
  -o gpurun_out/$TAG -f python tools/profile_step.py $N 4 1 0 3 > gpurun_out/ncu_$TAG.log 2>&1
python tools/ncu_summary.py gpurun_out/$TAG.ncu-rep > gpurun_out/${TAG}_summary.md 2>&1
true
