#!/bin/bash
# Where a dynamic block's cost goes: ncu --set full with source of K1 on C2 at the
# product split (500:8) and with blocks of 2 (500:2), exported per CUDA source line.
set -u
OUT=gpurun_out/${1:-r02ac}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
EXP=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so
for s in 500:8 500:2; do
  tag=b${s#*:}
  CHECL_LIB=$EXP CHECL_STATIC_PERMILLE=${s%:*} CHECL_DYN_BLOCK=${s#*:} CHECL_DYN_MIN_ROUNDS=0 timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel<.int.0" -s 2 -c 1 -o /tmp/k1_$tag -f python tools/exp_run.py --config C2 --reps 2 > $OUT/ncu_$tag.log 2>&1
  ncu -i /tmp/k1_$tag.ncu-rep --page source --csv --print-source cuda > $OUT/src_cuda_$tag.csv 2>&1
  ncu -i /tmp/k1_$tag.ncu-rep --page raw --csv > $OUT/raw_$tag.csv 2>&1
  python tools/ncu_summary.py /tmp/k1_$tag.ncu-rep > $OUT/summary_$tag.txt 2>&1
done
ls -la $OUT; head -20 $OUT/summary_b2.txt
