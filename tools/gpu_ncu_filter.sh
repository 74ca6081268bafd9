#!/bin/bash
# ncu --set full of k_filter at configs[2] (N molecules); summary + source csv
mkdir -p gpurun_out
N=${1:-1000000}
TAG=${2:-filt}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_filter" -c 1 \
  -o gpurun_out/$TAG -f python tools/profile_step.py $N 4 1 0 3 > gpurun_out/ncu_$TAG.log 2>&1
python tools/ncu_summary.py gpurun_out/$TAG.ncu-rep > gpurun_out/${TAG}_summary.md 2>&1
ncu -i gpurun_out/$TAG.ncu-rep --page details --csv > gpurun_out/${TAG}_details.csv 2>&1
ncu -i gpurun_out/$TAG.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/${TAG}_src.csv 2>&1
true
