#!/bin/bash
# r2 evidence on the final tree (profiles/r2): ncu capture of the bench kernels first (its summary feeds the
# bench's roofline; SKIP_CAPTURE=1 keeps the committed one), then the bench lines, the launch list of the
# default bench command and smoke()
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
if [ -z "$SKIP_CAPTURE" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sigmo_filter_lane_jit|k_join_lane" -s 6 -c 3 -o $O/ncu_full_L2 python tools/profile_step.py 1000000 2 1 0 3 > $O/ncu_full.log 2>&1
python tools/ncu_traffic.py $O/ncu_full_L2.ncu-rep 2 > $O/ncu_traffic.json && cp $O/ncu_traffic.json profiles/r2/ncu_traffic.json
fi
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 900 python bench.py --config 1 --steps 20 --warmup 3 --no-cpu-baseline > $O/bench_c1.json 2> $O/bench_c1.err
timeout 900 python bench.py --config 3 --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_c3.json 2> $O/bench_c3.err
timeout 1200 python bench.py --config 4 --steps 3 --warmup 3 --no-cpu-baseline > $O/bench_c4.json 2> $O/bench_c4.err
timeout 900 python bench.py --induced --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_c2_induced.json 2> $O/bench_c2_induced.err
timeout 900 python bench.py --ns --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/bench_c2_ns.json 2> $O/bench_c2_ns.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_bench_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/ncu_bench.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for f in $O/bench_*.json; do echo $f; head -c 300 $f; echo; done
tail -2 $O/smoke.log; cat $O/ncu_traffic.json | head -30
