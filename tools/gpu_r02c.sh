#!/bin/bash
# Full GPU round: tests, smoke, bench (C3 default + extras), ncu launch list of the
# bench, ncu --set full of K1/K2 on C3 and C2, the exact-incremental diff pass, the
# CRC-only pass and the peer-read K2 register path.
set -u
O=gpurun_out/${1:-r02c}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -4 $O/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
python -c "
import json;d=json.load(open('$O/bench.json'));r=d['roofline'];e=d['e2e']
print('C3 value %.1f step %.3f frac %.3f e2e %.2f' % (d['value'], d['ms_per_step'], r['frac'], e['value']))
for k,v in d['extras'].items(): print(k, v.get('value'), v.get('roofline',{}).get('frac'), v.get('error'))"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > $O/nvsmi.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-extras > $O/launches.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"tma_kernel" -s 2 -c 2 -o $O/prof -f python tools/profile_step.py --config C3 --reps 2 > $O/ncu_full.log 2>&1
tail -1 $O/ncu_full.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tma_kernel" -s 2 -c 2 -o $O/prof_c2 -f python tools/profile_step.py --config C2 --reps 2 > $O/ncu_full_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"diff_kernel|tma_kernel" -c 4 -o $O/prof_inc -f python bench.py --mode incremental --config C2 --steps 1 --warmup 1 --dirty 0.01 > $O/ncu_inc.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tma_kernel" -c 3 -o $O/prof_inc_crc -f python bench.py --mode incremental --config C2 --steps 1 --warmup 1 --dirty 0.01 --rule crc > $O/ncu_inc_crc.log 2>&1
CHECL_FORCE_IMAGE_REMOTE=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tma_kernel" -s 2 -c 2 -o $O/prof_remote -f python tools/profile_step.py --config C2 --reps 2 > $O/ncu_remote.log 2>&1
ls $O
