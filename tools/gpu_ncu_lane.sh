#!/bin/bash
# ncu --set full of k_filter_lane at configs[2] (1M molecules, L=4)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_filter_lane -s 2 -c 1 -o gpurun_out/${NCU_NAME:-filt_lane} python tools/profile_step.py 1000000 4 1 0 3 > gpurun_out/ncu_lane.log 2>&1
tail -3 gpurun_out/ncu_lane.log
