#!/bin/bash
# A/B: small host-image checkpoints with K1 storing into the mapped pinned image
# (default) vs the staged slot + D2H (CHECL_ZERO_COPY_MAX=0). GPU tests first.
set -u
O=gpurun_out/zc
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log; tail -2 $O/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; tail -1 $O/smoke.log
for rep in 1 2; do for zc in 0 8388608; do
  CHECL_ZERO_COPY_MAX=$zc timeout 300 python bench.py --config C1 --no-cpu-baseline --steps 50 > $O/c1_zc${zc}_$rep.json 2>/dev/null
  python -c "
import json
d=json.loads(open('$O/c1_zc${zc}_$rep.json').read().strip().splitlines()[-1]);e=d['e2e']
print('zc=$zc rep=$rep e2e %.2f GB/s checkpoint %.4f ms restore %.4f ms drain %.1f GB/s value %.1f' % (e['value'], e['checkpoint_ms'], e['restore_ms'], e['drain_GBs'], d['value']))"
done; done | tee $O/summary.txt
CHECL_TRACE=1 timeout 120 python tools/trace_step.py C1 6 host > $O/trace_c1_host.log 2>&1; tail -4 $O/trace_c1_host.log
for t in memcheck racecheck synccheck; do timeout 600 compute-sanitizer --tool $t python tools/sanitize.py > $O/san_$t.log 2>&1; echo "== $t"; grep -E "sanitize ok|SUMMARY" $O/san_$t.log; done | tee $O/sanitizer.txt
