#!/bin/bash
# ncu --set full of K1 (C2) for the previous build and the quad-chain build.
set -u
OUT=gpurun_out/${1:-r02l}
R=/tmp/ncu_r02l
mkdir -p $OUT $R
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for v in prev default; do
  if [ $v = default ]; then lib=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; else lib=$PWD/exp_libs/$v/libchecl.so; fi
  CHECL_LIB=$lib timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel<.int.0" -s 2 -c 1 -o $R/k1_$v -f python tools/exp_run.py --config C2 --reps 1 > $OUT/ncu_$v.log 2>&1
  python tools/ncu_summary.py $R/k1_$v.ncu-rep > $OUT/summary_$v.txt 2>&1
  ncu -i $R/k1_$v.ncu-rep --page source --csv --print-source sass > $OUT/sass_$v.csv 2>&1
done
cat $OUT/summary_*.txt
ls -la $OUT
