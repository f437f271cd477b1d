#!/bin/bash
# Quick GPU check: tests, smoke, C2/C1/C3 bench lines (x2), host trace of C2.
set -u
O=gpurun_out/${1:-q}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log; tail -2 $O/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; tail -1 $O/smoke.log
for rep in 1 2; do
  timeout 600 python bench.py > $O/c2_$rep.json 2> $O/c2_$rep.err
  timeout 300 python bench.py --config C1 --no-cpu-baseline > $O/c1_$rep.json 2>/dev/null
  timeout 600 python bench.py --config C3 --steps 5 --no-cpu-baseline > $O/c3_$rep.json 2>/dev/null
done
CHECL_TRACE=1 timeout 120 python tools/trace_step.py > $O/trace.log 2>&1
for f in $O/c*_*.json; do python -c "
import json
d=json.load(open('$f'));r=d['roofline'];e=d.get('e2e') or {}
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f e2e %.2f launches %d' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac'], e.get('value', 0), d['gpu_launches']))" 2>&1 | tail -1; done | tee $O/summary.txt
tail -4 $O/trace.log
