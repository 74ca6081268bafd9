#!/bin/bash
# one ncu --set full capture of the lane join (configs[2], L=2) under the name $NCU_NAME
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_join_lane -s ${NCU_S:-2} -c 2 -o gpurun_out/${NCU_NAME:-join_q} python tools/profile_step.py 1000000 2 1 0 3 > gpurun_out/ncu_join_q.log 2>&1
tail -2 gpurun_out/ncu_join_q.log
