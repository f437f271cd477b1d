#!/bin/bash
# 11 warps per CTA (the TMA kernel's tables + 11 x 2 tiles still fit 227 KiB) against
# the product's 10: parity of the w11 build (kernel shapes, parity, fuzz) and pack /
# verify / CRC-rule pass on C1, 64 MiB, 256 MiB, C2, C3.
set -u
OUT=gpurun_out/${1:-r02aa}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
W11=$PWD/exp_libs/w11/libchecl.so
CHECL_LIB=$W11 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_incremental.py -x -q > $OUT/pytest_w11.log 2>&1
tail -1 $OUT/pytest_w11.log
NEW=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so
for pass in 1 2 3; do
  for args in "--config C1 --reps 40" "--mib 64 --reps 30" "--mib 256 --reps 30" "--config C2 --reps 30" "--config C3 --reps 8"; do
    for v in w10 w11; do
      if [ $v = w11 ]; then lib=$W11; else lib=$NEW; fi
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$lib timeout 300 python tools/exp_run.py $args --incr >> $OUT/ab.txt 2>&1
    done
  done
done
cat $OUT/ab.txt
