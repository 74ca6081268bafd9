#!/bin/bash
# r2 evidence on the final tree (profiles/r2): bench lines, ncu captures, sanitizer, GPU suite
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 900 python bench.py --config 1 --steps 20 --warmup 3 --no-cpu-baseline > $O/bench_c1.json 2> $O/bench_c1.err
timeout 900 python bench.py --config 3 --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_c3.json 2> $O/bench_c3.err
timeout 1200 python bench.py --config 4 --steps 3 --warmup 3 --no-cpu-baseline > $O/bench_c4.json 2> $O/bench_c4.err
timeout 900 python bench.py --induced --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_c2_induced.json 2> $O/bench_c2_induced.err
timeout 900 python bench.py --ns --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/bench_c2_ns.json 2> $O/bench_c2_ns.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sigmo_filter_lane_jit|k_join_lane" -s 6 -c 3 -o $O/ncu_full_L2 python tools/profile_step.py 1000000 2 1 0 3 > $O/ncu_full.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_bench_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_bench.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_cases.py > $O/sanitizer_$tool.log 2>&1
  echo "rc=$?" >> $O/sanitizer_$tool.log
done
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for f in $O/bench_*.json; do echo $f; head -c 400 $f; echo; done
tail -3 $O/gputest.log; tail -2 $O/smoke.log
for tool in memcheck racecheck synccheck; do tail -2 $O/sanitizer_$tool.log; done
