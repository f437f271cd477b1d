#!/bin/bash
# GPU tests, smoke, C3 trace, quick benches
set -u
O=gpurun_out/${1:-r02i}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=5 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; tail -1 $O/smoke.log
CHECL_TRACE=1 timeout 300 python tools/trace_step.py C3 6 > $O/trace_c3.log 2>&1; tail -4 $O/trace_c3.log
for rep in 1 2; do
  timeout 600 python bench.py --no-cpu-baseline --no-extras > $O/c3_$rep.json 2>/dev/null
  timeout 300 python bench.py --config C2 --no-cpu-baseline --no-extras --no-e2e > $O/c2_$rep.json 2>/dev/null
done
for f in $O/c3_*.json $O/c2_*.json; do python -c "
import json
d=json.load(open('$f'));r=d['roofline'];e=d.get('e2e') or {}
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f e2e %.2f' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac'], e.get('value') or 0))" 2>&1 | tail -1; done | tee $O/quick.txt
