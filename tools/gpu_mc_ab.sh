#!/bin/bash
# Multicast table prologue (CHECL_TABLE_MC=1): GPU tests, sanitizer, A/B bench lines.
set -u
O=gpurun_out/${1:-mc}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
CHECL_TABLE_MC=1 timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_mc.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu_mc.log; tail -2 $O/pytest_gpu_mc.log
for tool in memcheck racecheck synccheck; do
  CHECL_TABLE_MC=1 CHECL_KERNEL=4 timeout 600 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}.log 2>&1
  echo "$tool: $(grep -E 'sanitize ok' $O/san_${tool}.log) $(grep -E 'SUMMARY' $O/san_${tool}.log)"
done | tee $O/sanitizer.txt
CHECL_TABLE_MC=1 CHECL_WARP_TRACE=1 timeout 120 python tools/profile_step.py --config C2 --reps 3 > $O/warp_trace_mc.txt 2>&1
for rep in 1 2 3; do for M in 0 1; do
  CHECL_TABLE_MC=$M timeout 300 python bench.py --no-cpu-baseline --no-e2e > $O/c2_m${M}_$rep.json 2>/dev/null
  CHECL_TABLE_MC=$M timeout 300 python bench.py --config C3 --steps 5 --no-cpu-baseline --no-e2e > $O/c3_m${M}_$rep.json 2>/dev/null
done; done
for f in $O/c*_m*.json; do python -c "
import json
d=json.load(open('$f'));r=d['roofline']
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac']))" 2>/dev/null; done | tee $O/ab.txt
grep "op 0" $O/warp_trace_mc.txt | tail -2
