#!/bin/bash
# iteration: gpu tests, configs[2] bench, ncu of the join at 200k molecules
bash tools/gpu_quick.sh
bash tools/gpu_ncu_join.sh 200000 ${1:-jiter}
