#!/bin/bash
# ncu --set full of the narrow lane join (Find All) at configs[2]
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_join_lane -s ${NCU_SKIP:-4} -c 1 -o gpurun_out/${NCU_NAME:-join} python tools/profile_step.py 1000000 4 1 ${MODE:-0} 3 > gpurun_out/ncu_join.log 2>&1
tail -2 gpurun_out/ncu_join.log
