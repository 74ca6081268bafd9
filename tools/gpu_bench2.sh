for i in 1 2; do timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b2_$i.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/b2_$i.json')); print(d['ms_per_step'], d['stage_ms'], d['find_first']['ms_per_step'], d['clocks'])"; done
SIGMO_FILTER_JIT=0 timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b2_g.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/b2_g.json')); print('generic', d['ms_per_step'], d['stage_ms'], d['find_first']['ms_per_step'])"
