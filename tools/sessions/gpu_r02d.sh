#!/bin/bash
# tests + smoke, then ncu captures reduced to CSV summaries on the box (the .ncu-rep
# files stay there: gpurun_out must stay under 64 MiB)
set -u
O=gpurun_out/${1:-r02d}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=10 ${2:-} > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -4 $O/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; tail -1 $O/smoke.log
R=/tmp/ncu_$$
mkdir -p $R
cap() {  # name, kernel regex, "ncu extra args", command...
  local name=$1 rx=$2 extra=$3; shift 3
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$rx" $extra -o $R/$name -f "$@" > $O/ncu_$name.log 2>&1
  ncu -i $R/$name.ncu-rep --page raw --csv > $O/${name}_raw.csv 2>/dev/null
  ncu -i $R/$name.ncu-rep --page details --csv > $O/${name}_details.csv 2>/dev/null
  python tools/ncu_summary.py $R/$name.ncu-rep > $O/${name}_summary.txt 2>&1
}
cap c3 tma_kernel "-s 2 -c 2" python tools/profile_step.py --config C3 --reps 2
cap c2 tma_kernel "-s 2 -c 2" python tools/profile_step.py --config C2 --reps 2
cap inc_bytes "diff_kernel|sweep_kernel|snapshot_kernel" "-c 6" python bench.py --mode incremental --config C2 --steps 1 --warmup 1 --dirty 0.01
cap inc_crc "tma_kernel" "-c 3" python bench.py --mode incremental --config C2 --steps 1 --warmup 1 --dirty 0.01 --rule crc
export CHECL_FORCE_IMAGE_REMOTE=1; cap remote tma_kernel "-s 2 -c 2" python tools/profile_step.py --config C2 --reps 2; unset CHECL_FORCE_IMAGE_REMOTE
timeout 300 python tools/mem_diag.py > $O/mem_diag.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-extras > $O/launches.log 2>&1
CHECL_TRACE=1 timeout 300 python tools/trace_step.py C3 6 > $O/trace_c3.log 2>&1
CHECL_TRACE=1 timeout 120 python tools/trace_step.py C2 6 > $O/trace_c2.log 2>&1
du -sh $O
for rep in 1 2; do
  timeout 600 python bench.py --no-cpu-baseline --no-extras > $O/c3_$rep.json 2>/dev/null
  timeout 300 python bench.py --config C2 --no-cpu-baseline --no-extras > $O/c2_$rep.json 2>/dev/null
done
for f in $O/c3_*.json $O/c2_*.json; do python -c "
import json
d=json.load(open('$f'));r=d['roofline'];e=d.get('e2e') or {}
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f e2e %.2f' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac'], e.get('value', 0)))" 2>&1 | tail -1; done | tee $O/quick.txt
