#!/bin/bash
# Round-2 evidence session: tests, smoke, the default bench line (C3 + extras + oracle
# baseline), the reference arm, ncu launch list of the bench command, ncu --set full of
# K1/K2 on C3 (traffic), incremental and migration lines, C1, host traces.
set -u
O=gpurun_out/${1:-r02_final}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; tail -1 $O/smoke.log
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > $O/nvsmi.txt
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err
python -c "
import json;d=json.load(open('$O/bench.json'));r=d['roofline'];e=d['e2e']
print('C3 value %.1f step %.3f frac %.3f traffic %s e2e %.2f launches %d' % (d['value'], d['ms_per_step'], r['frac'], r['traffic'], e['value'], d['gpu_launches']))
for k,v in d['extras'].items(): print(k, v.get('value'), v.get('roofline',{}).get('frac'), v.get('error'))"
timeout 600 python bench.py --config C1 --no-cpu-baseline --no-extras > $O/bench_c1.json 2> $O/bench_c1.err
timeout 600 python bench.py --config C5 > $O/bench_c5.json 2> $O/bench_c5.err
timeout 600 python bench.py --config C5 --c5-large > $O/bench_c5_large.json 2> $O/bench_c5_large.err
for cfg in C3 C2; do for rule in bytes crc; do for d in 0.01 0.1; do
  timeout 600 python bench.py --mode incremental --config $cfg --dirty $d --rule $rule > $O/inc_${cfg}_${rule}_$d.json 2> /dev/null
done; done; done
CHECL_TRACE=1 timeout 300 python tools/trace_step.py C3 6 > $O/trace_c3.log 2>&1
CHECL_TRACE=1 timeout 120 python tools/trace_step.py C2 6 > $O/trace_c2.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"tma_kernel|sweep_kernel|balanced_kernel|snapshot_kernel|expand_plan|build_tables|meta_crc" -c 60 --csv --log-file $O/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-extras --no-e2e > $O/launches.log 2>&1
R=/tmp/ncu_$$; mkdir -p $R
timeout 1200 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel|meta_crc" -c 6 -o $R/c3 -f python tools/profile_step.py --config C3 --reps 2 > $O/ncu_c3.log 2>&1
python tools/ncu_summary.py $R/c3.ncu-rep > $O/c3_summary.txt 2>&1
ncu -i $R/c3.ncu-rep --page details --csv > $O/c3_details.csv 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel" -c 4 -o $R/c2 -f python tools/profile_step.py --config C2 --reps 2 > $O/ncu_c2.log 2>&1
python tools/ncu_summary.py $R/c2.ncu-rep > $O/c2_summary.txt 2>&1
ncu -i $R/c2.ncu-rep --page raw --csv --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum > $O/c2_dram.csv 2>&1
du -sh $O
