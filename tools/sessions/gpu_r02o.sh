#!/bin/bash
# Work-split sweep after the asynchronous block fetch: static share x dynamic block
# size for the previous commit's experiments build (base_exp) and the new one, on C2,
# one 256 MiB buffer (dynamic tail forced on: CHECL_DYN_MIN_ROUNDS=0) and C3.
set -u
OUT=gpurun_out/${1:-r02o}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
NEW=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so
BASE=$PWD/exp_libs/base_exp/libchecl.so
run() {  # lib tag pm blk args...
  local lib=$1 tag=$2 pm=$3 blk=$4; shift 4
  echo -n "$tag pm=$pm blk=$blk " >> $OUT/sweep.txt
  CHECL_LIB=$lib CHECL_STATIC_PERMILLE=$pm CHECL_DYN_BLOCK=$blk CHECL_DYN_MIN_ROUNDS=0 timeout 300 python tools/exp_run.py "$@" >> $OUT/sweep.txt 2>&1
}
for pass in 1 2; do
  for spec in 750:8 500:8 500:4 250:4 0:8 0:4 0:2 500:2 900:4; do
    pm=${spec%:*}; blk=${spec#*:}
    run $BASE base $pm $blk --config C2 --reps 20
    run $NEW new $pm $blk --config C2 --reps 20
    run $BASE base $pm $blk --mib 256 --reps 20
    run $NEW new $pm $blk --mib 256 --reps 20
  done
done
for spec in 750:8 500:4 0:4; do
  pm=${spec%:*}; blk=${spec#*:}
  run $BASE base $pm $blk --config C3 --reps 6
  run $NEW new $pm $blk --config C3 --reps 6
done
cat $OUT/sweep.txt
