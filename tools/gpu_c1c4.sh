#!/bin/bash
# C4 at full size (restart mode) + C1 latency anatomy (warp trace, ncu full of K1/K2).
# usage: tools/gpu_c1c4.sh <tag>
set -u
TAG=${1:-r}
O=gpurun_out/$TAG
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python bench.py --config C4 --steps 3 --warmup 3 > $O/bench_c4.json 2> $O/bench_c4.err; tail -c 400 $O/bench_c4.json
CHECL_WARP_TRACE=1 timeout 120 python tools/profile_step.py --config C1 --reps 6 --flush --verbose > $O/warp_trace_c1.txt 2>&1
CHECL_WARP_TRACE=1 timeout 120 python tools/profile_step.py --config C1 --reps 6 --verbose > $O/warp_trace_c1_warm.txt 2>&1
CHECL_TRACE=1 timeout 120 python tools/trace_step.py C1 6 > $O/trace_c1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"balanced_kernel|tma_kernel" -s 4 -c 2 -o $O/prof_c1 -f python tools/profile_step.py --config C1 --reps 4 --flush > $O/ncu_c1.log 2>&1
tail -1 $O/ncu_c1.log
