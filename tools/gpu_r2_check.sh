#!/bin/bash
# full GPU suite, sanitizer (memcheck/racecheck/synccheck over tools/sanitize_cases.py), one default bench
mkdir -p gpurun_out/check
O=gpurun_out/check
timeout 2400 python -m pytest tests -m gpu -q --durations=12 > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_cases.py > $O/sanitizer_$tool.log 2>&1
  echo "rc=$?" >> $O/sanitizer_$tool.log
done
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 2 > $O/bench.json 2> $O/bench.err
tail -15 $O/gputest.log
for tool in memcheck racecheck synccheck; do tail -3 $O/sanitizer_$tool.log; done
python -c "
import json; d=json.load(open('$O/bench.json')); print(d['ms_per_step'], d['value'], d['stage_ms'], d['find_first'], d['e2e']['value'], d['clocks'])" || tail -5 $O/bench.err
