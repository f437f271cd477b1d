#!/bin/bash
# In-CTA column tables + size-dependent work split: parity, product A/B against the
# previous commit (exp_libs/base), the table change alone (experiments builds with
# the split pinned), warp trace, and the remaining split points at C3 / 4 GiB.
set -u
OUT=gpurun_out/${1:-r02q}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_incremental.py -x -q > $OUT/pytest.log 2>&1
tail -3 $OUT/pytest.log
NEW=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so
BASE=$PWD/exp_libs/base/libchecl.so
NEWX=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so
BASEX=$PWD/exp_libs/base_exp/libchecl.so
for pass in 1 2 3; do
  for args in "--config C2 --reps 30" "--mib 64 --reps 30" "--mib 128 --reps 30" "--mib 256 --reps 30" "--config C3 --reps 8" "--mib 4096 --reps 6"; do
    for v in base new; do
      if [ $v = new ]; then lib=$NEW; else lib=$BASE; fi
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$lib timeout 300 python tools/exp_run.py $args >> $OUT/ab.txt 2>&1
    done
  done
done
for pass in 1 2; do
  for s in 750:8 500:8; do
    for v in base new; do
      if [ $v = new ]; then lib=$NEWX; else lib=$BASEX; fi
      echo -n "$v pm=${s%:*} blk=${s#*:} " >> $OUT/tables_ab.txt
      CHECL_LIB=$lib CHECL_STATIC_PERMILLE=${s%:*} CHECL_DYN_BLOCK=${s#*:} CHECL_DYN_MIN_ROUNDS=0 timeout 300 python tools/exp_run.py --config C2 --reps 30 --incr >> $OUT/tables_ab.txt 2>&1
    done
  done
done
for s in 600:8 500:8 750:8; do
  for args in "--config C3 --reps 6" "--mib 4096 --reps 6"; do
    echo -n "pm=${s%:*} blk=${s#*:} " >> $OUT/split_large.txt
    CHECL_LIB=$NEWX CHECL_STATIC_PERMILLE=${s%:*} CHECL_DYN_BLOCK=${s#*:} CHECL_DYN_MIN_ROUNDS=0 timeout 300 python tools/exp_run.py $args >> $OUT/split_large.txt 2>&1
  done
done
CHECL_LIB=$NEWX CHECL_WARP_TRACE=1 timeout 300 python tools/trace_step.py C2 4 > $OUT/warp_trace_new.txt 2>&1
cat $OUT/ab.txt $OUT/tables_ab.txt $OUT/split_large.txt; grep "kernel 4" $OUT/warp_trace_new.txt | head -8
