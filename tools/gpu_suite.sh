#!/bin/bash
# full GPU suite with per-test durations
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --durations=25 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/suite.log 2>&1; echo "pytest rc=$?" >> gpurun_out/suite.log
tail -40 gpurun_out/suite.log
