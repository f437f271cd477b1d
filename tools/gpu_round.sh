#!/bin/bash
# One GPU session: tests, bench, launch list, full ncu capture of K1 and K2.
# usage: tools/gpu_round.sh <tag> [pytest-args]
set -u
TAG=${1:-r}
mkdir -p gpurun_out/$TAG
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/$TAG/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q ${2:-} > gpurun_out/$TAG/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/$TAG/pytest_gpu.log
tail -5 gpurun_out/$TAG/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/$TAG/smoke.log 2>&1; tail -1 gpurun_out/$TAG/smoke.log
timeout 600 python bench.py > gpurun_out/$TAG/bench.json 2> gpurun_out/$TAG/bench.err; tail -c 600 gpurun_out/$TAG/bench.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/$TAG/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/$TAG/launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:snapshot_kernel -s 2 -c 2 -o gpurun_out/$TAG/prof -f python tools/profile_step.py --reps 2 > gpurun_out/$TAG/ncu_full.log 2>&1
tail -2 gpurun_out/$TAG/ncu_full.log
