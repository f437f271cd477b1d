#!/bin/bash
# Tail blocks: the last (rounds per warp x warps) dynamic rounds in smaller blocks
# (experiments build, CHECL_TAIL_RPW / CHECL_TAIL_BLOCK) on C2, 256 MiB and C3, with
# the product's split for each; kernel-shape parity with a tail forced on first.
set -u
OUT=gpurun_out/${1:-r02r}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
EXP=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so
CHECL_LIB=$EXP CHECL_TAIL_RPW=4 CHECL_TAIL_BLOCK=2 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -x -q > $OUT/pytest_tail.log 2>&1
tail -2 $OUT/pytest_tail.log
for pass in 1 2; do
  for s in 0:0 2:2 4:2 4:4 8:4 2:1 8:2 16:4; do
    for args in "--config C2 --reps 30" "--mib 256 --reps 30" "--config C3 --reps 6"; do
      echo -n "tail=$s " >> $OUT/sweep.txt
      CHECL_LIB=$EXP CHECL_TAIL_RPW=${s%:*} CHECL_TAIL_BLOCK=${s#*:} timeout 300 python tools/exp_run.py $args >> $OUT/sweep.txt 2>&1
    done
  done
done
cat $OUT/sweep.txt
