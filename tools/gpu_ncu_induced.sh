#!/bin/bash
# ncu --set full of the induced-mode lane join (k_join_lane<2,false>) at configs[2], 1M molecules
mkdir -p gpurun_out
SIGMO_PROFILE_INDUCED=1 timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_join_lane" -c 1 \
  -o gpurun_out/join_ind -f python tools/profile_step.py 1000000 4 1 0 3 > gpurun_out/ncu_join_ind.log 2>&1
python tools/ncu_summary.py gpurun_out/join_ind.ncu-rep > gpurun_out/join_ind_summary.md 2>&1
tail -3 gpurun_out/ncu_join_ind.log
head -40 gpurun_out/join_ind_summary.md
