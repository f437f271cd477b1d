#!/bin/bash
# Graph vs stream timed launches: GPU tests, then A/B bench lines (CHECL_GRAPH=0|1).
# usage: tools/gpu_graph_ab.sh <tag>
set -u
TAG=${1:-r}
O=gpurun_out/$TAG
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/pytest_gpu.log
CHECL_GRAPH=0 timeout 120 python -m pytest tests/test_gpu_parity.py tests/test_gpu_kernels.py -m gpu -x -q > $O/pytest_gpu_nograph.log 2>&1; tail -1 $O/pytest_gpu_nograph.log
for rep in 1 2; do
for G in 0 1; do
  CHECL_GRAPH=$G timeout 300 python bench.py --no-cpu-baseline --no-e2e > $O/c2_g${G}_$rep.json 2> $O/c2_g${G}_$rep.err
  CHECL_GRAPH=$G timeout 300 python bench.py --config C1 --no-cpu-baseline --no-e2e > $O/c1_g${G}_$rep.json 2> $O/c1_g${G}_$rep.err
  CHECL_GRAPH=$G timeout 300 python bench.py --config C3 --steps 5 --no-cpu-baseline --no-e2e > $O/c3_g${G}_$rep.json 2> $O/c3_g${G}_$rep.err
done
done
for G in 0 1; do
  CHECL_GRAPH=$G timeout 300 python bench.py --no-cpu-baseline > $O/c2e2e_g${G}.json 2> $O/c2e2e_g${G}.err
done
CHECL_TRACE=1 timeout 120 python tools/trace_step.py C1 6 > $O/trace_c1.log 2>&1
CHECL_TRACE=1 timeout 120 python tools/trace_step.py C2 6 > $O/trace_c2.log 2>&1
CHECL_TRACE=1 timeout 300 python bench.py --restart --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $O/c2_restart_trace.json 2> $O/c2_restart_trace.err
python - <<'PY'
import json, glob, os
O = os.environ.get("O", "")
PY
for f in $O/c*_g*.json; do python -c "
import json,sys
d=json.load(open('$f'));r=d['roofline'];e=d.get('e2e') or {}
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f e2e %s' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac'], e.get('value')))" 2>/dev/null; done | tee $O/ab.txt
