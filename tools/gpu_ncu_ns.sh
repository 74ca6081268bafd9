#!/bin/bash
mkdir -p gpurun_out
SIGMO_PROFILE_NS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_support_lane -s 2 -c 1 -o gpurun_out/${NCU_NAME:-ns} python tools/profile_step.py 1000000 4 1 0 3 > gpurun_out/ncu_ns.log 2>&1
tail -2 gpurun_out/ncu_ns.log
