#!/bin/bash
# ncu --set full of k_filter and k_join_lane (Find All) at configs[2] with N molecules; raw + source csv pages
mkdir -p gpurun_out
N=${1:-1000000}
TAG=${2:-full}
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_filter|k_join_lane" -c 2 \
  -o gpurun_out/$TAG -f python tools/profile_step.py $N 4 1 0 3 > gpurun_out/ncu_$TAG.log 2>&1
python tools/ncu_summary.py gpurun_out/$TAG.ncu-rep > gpurun_out/${TAG}_summary.md 2>&1
ncu -i gpurun_out/$TAG.ncu-rep --page raw --csv > gpurun_out/${TAG}_raw.csv 2>&1
ncu -i gpurun_out/$TAG.ncu-rep --page details --csv > gpurun_out/${TAG}_details.csv 2>&1
for k in k_filter k_join_lane; do
  ncu -i gpurun_out/$TAG.ncu-rep -k regex:$k --page source --csv --print-source cuda,sass > gpurun_out/${TAG}_src_$k.csv 2>&1
done
true
