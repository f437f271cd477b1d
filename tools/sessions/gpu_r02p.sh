#!/bin/bash
# Static share / dynamic block size per launch size (experiments build): which
# absolute amount of dynamic rounds per warp is best at 64 MiB .. C3 / 4 GiB.
set -u
OUT=gpurun_out/${1:-r02p}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
EXP=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so
run() {  # pm blk args...
  local pm=$1 blk=$2; shift 2
  echo -n "pm=$pm blk=$blk " >> $OUT/sweep.txt
  CHECL_LIB=$EXP CHECL_STATIC_PERMILLE=$pm CHECL_DYN_BLOCK=$blk CHECL_DYN_MIN_ROUNDS=0 timeout 300 python tools/exp_run.py "$@" >> $OUT/sweep.txt 2>&1
}
for pass in 1 2; do
  for s in 1000:8 640:2 500:2 640:4 500:4; do run ${s%:*} ${s#*:} --mib 64 --reps 30; done
  for s in 1000:8 500:4 640:4 250:4 500:2 750:4; do run ${s%:*} ${s#*:} --mib 128 --reps 30; done
  for s in 500:4 640:4 360:4 500:8; do run ${s%:*} ${s#*:} --mib 256 --reps 30; done
  for s in 500:8 600:8 400:8 750:8 500:6 600:4; do run ${s%:*} ${s#*:} --config C2 --reps 30; done
  for s in 750:8 850:8 900:8 950:8 900:16; do run ${s%:*} ${s#*:} --config C3 --reps 6; done
  for s in 750:8 900:8 950:8; do run ${s%:*} ${s#*:} --mib 4096 --reps 6; done
done
cat $OUT/sweep.txt
