mkdir -p gpurun_out/c1ab
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c1ab/build.log 2>&1
for rep in 1 2; do for k in 0 2 3 4; do
  CHECL_KERNEL=$k timeout 300 python bench.py --config C1 --no-cpu-baseline --no-e2e --steps 50 > gpurun_out/c1ab/c1_k${k}_$rep.json 2>/dev/null
  python -c "
import json
d=json.loads(open('gpurun_out/c1ab/c1_k${k}_$rep.json').read().strip().splitlines()[-1]);r=d['roofline']
print('k=$k rep=$rep value %.1f step %.4f ms pack %.2f us verify %.2f us' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3))"
done; done | tee gpurun_out/c1ab/summary.txt
