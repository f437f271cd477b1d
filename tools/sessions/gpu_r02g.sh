#!/bin/bash
# carveout microbench, CRC-only pass + K1 source-level ncu, Eq. (1) on disk, C3 trace, quick bench
set -u
O=gpurun_out/${1:-r02g}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/carveout tools/microbench/carveout.cu && /tmp/carveout > $O/carveout.txt 2>&1; cat $O/carveout.txt
R=/tmp/ncu_$$; mkdir -p $R
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel<2" -c 2 -o $R/crc -f python bench.py --mode incremental --config C2 --steps 1 --warmup 1 --dirty 0.01 --rule crc > $O/ncu_crc.log 2>&1
python tools/ncu_summary.py $R/crc.ncu-rep > $O/crc_summary.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel<0" -s 1 -c 1 -o $R/k1 -f python tools/profile_step.py --config C2 --reps 2 > $O/ncu_k1.log 2>&1
ncu -i $R/k1.ncu-rep --page source --csv --print-source sass > $O/k1_source_sass.csv 2>&1
timeout 1500 python tools/cost_model.py --dir $PWD --reps 5 > $O/cost_model_disk.json 2> $O/cost_model_disk.err; echo "cost disk rc=$?"
CHECL_TRACE=1 timeout 300 python tools/trace_step.py C3 6 > $O/trace_c3.log 2>&1; tail -2 $O/trace_c3.log
for rep in 1 2; do
  timeout 600 python bench.py --no-cpu-baseline --no-extras > $O/c3_$rep.json 2>/dev/null
done
for f in $O/c3_*.json; do python -c "
import json
d=json.load(open('$f'));r=d['roofline'];e=d.get('e2e') or {}
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f e2e %.2f' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac'], e.get('value', 0)))" 2>&1 | tail -1; done | tee $O/quick.txt
du -sh $O
