#!/bin/bash
# One GPU session: tests, smoke, bench (C2 + C1 + C3), launch list, full ncu capture
# of K1 and K2 on C2. usage: tools/gpu_round.sh <tag> [pytest-args]
set -u
TAG=${1:-r}
O=gpurun_out/$TAG
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q ${2:-} > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err; tail -c 300 $O/bench.json
timeout 300 python bench.py --config C1 --no-cpu-baseline > $O/bench_c1.json 2> $O/bench_c1.err
timeout 900 python bench.py --config C3 --no-cpu-baseline --steps 5 > $O/bench_c3.json 2> $O/bench_c3.err
timeout 300 python bench.py --kind float --no-cpu-baseline --no-e2e > $O/bench_float.json 2> $O/bench_float.err
timeout 300 python bench.py --kind zeros --no-cpu-baseline --no-e2e > $O/bench_zeros.json 2> $O/bench_zeros.err
timeout 600 python bench.py --config C5 > $O/bench_c5.json 2> $O/bench_c5.err
timeout 300 python bench.py --mode incremental --dirty 0.01 > $O/bench_incremental_0.01.json 2> $O/bench_inc1.err
timeout 300 python bench.py --mode incremental --dirty 0.1 > $O/bench_incremental_0.1.json 2> $O/bench_inc10.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_ref.err
CHECL_TRACE=1 timeout 120 python tools/trace_step.py > $O/trace.log 2>&1
CHECL_TRACE=1 timeout 300 python tools/trace_step.py C3 6 > $O/trace_c3.log 2>&1
timeout 300 python bench.py --restart --no-cpu-baseline > $O/bench_c2_restart.json 2> $O/bench_c2_restart.err
timeout 1200 python bench.py --config C4 --steps 3 --warmup 3 > $O/bench_c4.json 2> $O/bench_c4.err
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > $O/nvsmi.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $O/launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"snapshot_kernel|balanced_kernel|tma_kernel" -s 2 -c 2 -o $O/prof -f python tools/profile_step.py --reps 2 > $O/ncu_full.log 2>&1
tail -1 $O/ncu_full.log
