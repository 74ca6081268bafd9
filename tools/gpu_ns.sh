#!/bin/bash
# neighbour-support tests + bench with and without the flag (configs[2])
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "neighbour or fig3 or c1_bitmap or enumerate" > gpurun_out/ns_test.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ns_test.log
tail -3 gpurun_out/ns_test.log
for ns in "" "--ns"; do
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 $ns > gpurun_out/ns_b$ns.json 2> gpurun_out/ns_b$ns.err
  python -c "
import json; d=json.load(open('gpurun_out/ns_b$ns.json')); print('$ns', d['ms_per_step'], d['stage_ms'], d['counts'], d['find_first']['ms_per_step'])" || tail -5 gpurun_out/ns_b$ns.err
done
