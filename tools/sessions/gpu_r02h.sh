#!/bin/bash
# commit breakdown trace, CRC-only pass + K1 source ncu, quick C3 bench, sanitizers + 400-case fuzz
set -u
O=gpurun_out/${1:-r02h}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
CHECL_TRACE=1 timeout 300 python tools/trace_step.py C3 6 > $O/trace_c3.log 2>&1; tail -3 $O/trace_c3.log
for rep in 1 2; do
  timeout 600 python bench.py --no-cpu-baseline --no-extras > $O/c3_$rep.json 2>/dev/null
done
for f in $O/c3_*.json; do python -c "
import json
d=json.load(open('$f'));r=d['roofline'];e=d.get('e2e') or {}
print('$f'.split('/')[-1], 'value %.1f step %.4f ms pack %.1f us verify %.1f us frac %.3f e2e %.2f drain %.3f fill %.3f' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3, r['frac'], e.get('value', 0), e.get('drain_frac_of_pcie',0), e.get('fill_frac_of_pcie',0)))" 2>&1 | tail -1; done | tee $O/quick.txt
R=/tmp/ncu_$$; mkdir -p $R
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel<.int.2" -c 2 -o $R/crc -f python bench.py --mode incremental --config C2 --steps 1 --warmup 1 --dirty 0.01 --rule crc > $O/ncu_crc.log 2>&1
python tools/ncu_summary.py $R/crc.ncu-rep > $O/crc_summary.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel<.int.0" -s 1 -c 1 -o $R/k1 -f python tools/profile_step.py --config C2 --reps 2 > $O/ncu_k1.log 2>&1
ncu -i $R/k1.ncu-rep --page source --csv --print-source sass > $O/k1_source_sass.csv 2>&1
bash tools/sessions/gpu_final_checks.sh ${1:-r02h}
du -sh $O
