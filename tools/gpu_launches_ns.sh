#!/bin/bash
mkdir -p gpurun_out
SIGMO_PROFILE_NS=1 timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_ns.csv python tools/profile_step.py 1000000 4 1 0 3 > gpurun_out/launches_ns.log 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/launches_ns.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
for r in rows[1:]:
    print(r[ki][:60], r[vi])
PY
