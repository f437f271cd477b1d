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
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > $O/nvsmi.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $O/launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"snapshot_kernel|balanced_kernel" -s 2 -c 2 -o $O/prof -f python tools/profile_step.py --reps 2 > $O/ncu_full.log 2>&1
tail -1 $O/ncu_full.log
