#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c2_full or c3_bench or random_tiny or fig3 or edge or c1_bitmap" > gpurun_out/pytest_p.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_p.log
tail -2 gpurun_out/pytest_p.log
SIGMO_FILTER_ROWS_GLOBAL=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c2_full or random_tiny or fig3 or edge or c1_bitmap" > gpurun_out/pytest_rg.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_rg.log
tail -2 gpurun_out/pytest_rg.log
bash tools/gpu_variants.sh
SIGMO_FILTER_ROWS_GLOBAL=1 bash tools/gpu_variants.sh
