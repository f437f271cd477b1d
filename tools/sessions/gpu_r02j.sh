#!/bin/bash
# Column-chain A/B (kColChains 1/2/4/8): parity of the default build, then pack /
# verify / CRC-rule pass timings per variant on C2 and C3.
set -u
OUT=gpurun_out/${1:-r02j}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_kernels.py tests/test_gpu_incremental.py tests/test_gpu_fuzz.py -x -q > $OUT/pytest.log 2>&1
tail -3 $OUT/pytest.log
for cfg in C2 C3; do
  reps=20; [ $cfg = C3 ] && reps=6
  for pass in 1 2; do
    for v in c1 c2 default c8; do
      if [ $v = default ]; then lib=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; else lib=$PWD/exp_libs/$v/libchecl.so; fi
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$lib timeout 300 python tools/exp_run.py --config $cfg --reps $reps --incr >> $OUT/ab.txt 2>&1
    done
  done
done
cat $OUT/ab.txt
