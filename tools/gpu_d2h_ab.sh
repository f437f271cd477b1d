#!/bin/bash
# Page-aligned split drain copies: GPU tests, then e2e A/B (CHECL_D2H_SPLIT=0|1), C3 and C2.
set -u
O=gpurun_out/${1:-d2h}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log; tail -2 $O/pytest_gpu.log
for rep in 1 2 3; do for S in 0 1; do
  CHECL_D2H_SPLIT=$S CHECL_STAGE_TRACE=1 timeout 300 python tools/profile_step.py --config C3 --host --reps 3 2>&1 | grep stages | tail -2 | sed "s/^/split=$S C3 /" >> $O/ab.txt
  CHECL_D2H_SPLIT=$S CHECL_STAGE_TRACE=1 timeout 300 python tools/profile_step.py --config C2 --host --reps 3 2>&1 | grep stages | tail -2 | sed "s/^/split=$S C2 /" >> $O/ab.txt
done; done
for S in 0 1; do CHECL_D2H_SPLIT=$S timeout 600 python bench.py --config C3 --steps 5 --no-cpu-baseline > $O/c3_s$S.json 2>/dev/null; done
for f in $O/c3_s*.json; do python -c "
import json;d=json.load(open('$f'));e=d['e2e'];print('$f', round(e['value'],2), round(e['checkpoint_GBs'],2), round(e['drain_frac_of_pcie'],3))"; done >> $O/ab.txt
cat $O/ab.txt | cut -c1-200
