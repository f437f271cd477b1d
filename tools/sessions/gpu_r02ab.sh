#!/bin/bash
# Column-kernel folds on the ALU (compile-time constant multiplies instead of
# conflicted shared-table lookups): parity, product A/B against the previous commit (exp_libs/prev3) on
# C2 / 256 MiB / C3, then finer dynamic blocks with both experiments builds.
set -u
OUT=gpurun_out/${1:-r02z}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_incremental.py -x -q > $OUT/pytest.log 2>&1
tail -2 $OUT/pytest.log
NEW=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so
OLD=$PWD/exp_libs/prev3/libchecl.so
NEWX=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so
OLDX=$PWD/exp_libs/prev3_exp/libchecl.so
for pass in 1 2 3; do
  for args in "--config C2 --reps 30" "--mib 256 --reps 30" "--config C3 --reps 8"; do
    for v in old new; do
      if [ $v = new ]; then lib=$NEW; else lib=$OLD; fi
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$lib timeout 300 python tools/exp_run.py $args --incr >> $OUT/ab.txt 2>&1
    done
  done
done
cat $OUT/ab.txt
for pass in 1 2; do
  for s in 500:8 500:4 500:2 250:4 750:4; do
    for v in old new; do
      if [ $v = new ]; then lib=$NEWX; else lib=$OLDX; fi
      echo -n "$v pm=${s%:*} blk=${s#*:} " >> $OUT/blocks.txt
      CHECL_LIB=$lib CHECL_STATIC_PERMILLE=${s%:*} CHECL_DYN_BLOCK=${s#*:} CHECL_DYN_MIN_ROUNDS=0 timeout 300 python tools/exp_run.py --config C2 --reps 30 >> $OUT/blocks.txt 2>&1
    done
  done
done
cat $OUT/blocks.txt
