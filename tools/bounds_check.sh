#!/bin/bash
# Device-side bounds checks in place of compute-sanitizer (closed on this pool): the GPU suite (without the
# full-size files unless FULL=1) and tools/sanitize_cases.py against a SIGMO_BOUNDS_CHECK build of libsigmo
# (built here by tools/build_variant.py into build/variants/bounds; an index out of its array traps the kernel)
mkdir -p gpurun_out/bounds
O=gpurun_out/bounds
export SIGMO_LIB=build/variants/bounds/libsigmo.so
K="not fullsize"
[ -n "$FULL" ] && K=""
timeout 2400 python -m pytest tests -m gpu -q ${K:+-k "$K"} > $O/gputest.log 2>&1; echo "pytest rc=$?" >> $O/gputest.log
timeout 900 python tools/sanitize_cases.py > $O/cases.log 2>&1; echo "cases rc=$?" >> $O/cases.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/bench.json 2> $O/bench.err; echo "bench rc=$?" >> $O/bench.err
tail -3 $O/gputest.log; tail -2 $O/cases.log; tail -1 $O/bench.err
