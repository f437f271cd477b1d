#!/bin/bash
# One-probe find_chunk: GPU tests, setup trace, A/B against the previous library (exp_libs/old).
set -u
O=gpurun_out/${1:-fc}
mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log; tail -2 $O/pytest_gpu.log
CHECL_LIB=$PWD/exp_libs/setup/libchecl.so CHECL_WARP_TRACE=1 timeout 120 python tools/profile_step.py --config C2 --reps 4 2>&1 | grep "op " > $O/setup_trace.txt
tail -2 $O/setup_trace.txt
for rep in 1 2 3; do
  for L in old new; do
    LIB=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; [ $L = old ] && LIB=$PWD/exp_libs/old/libchecl.so
    CHECL_LIB=$LIB timeout 300 python bench.py --no-cpu-baseline --no-e2e > $O/c2_${L}_$rep.json 2>/dev/null
    CHECL_LIB=$LIB timeout 300 python bench.py --config C3 --steps 5 --no-cpu-baseline --no-e2e > $O/c3_${L}_$rep.json 2>/dev/null
    CHECL_LIB=$LIB timeout 300 python bench.py --config C1 --no-cpu-baseline --no-e2e > $O/c1_${L}_$rep.json 2>/dev/null
  done
done
for f in $O/c*_*_*.json; do python -c "
import json
d=json.load(open('$f'));r=d['roofline']
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac']))" 2>/dev/null; done | sort | tee $O/ab.txt
