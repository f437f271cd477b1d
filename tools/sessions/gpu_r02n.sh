#!/bin/bash
# Asynchronous dynamic-block fetch A/B: parity of the new build (kernel-shape, parity,
# fuzz), pack / verify timings of exp_libs/base (the previous commit) against the new
# library on C2 and C3 (interleaved, two passes), warp traces of both, and the size
# scan with torch's copy_ of the same size beside each pack / verify.
set -u
OUT=gpurun_out/${1:-r02n}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_incremental.py -x -q > $OUT/pytest.log 2>&1
tail -3 $OUT/pytest.log
NEW=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so
for cfg in C2 C3; do
  reps=30; [ $cfg = C3 ] && reps=8
  for pass in 1 2 3; do
    for v in base new; do
      if [ $v = new ]; then lib=$NEW; else lib=$PWD/exp_libs/$v/libchecl.so; fi
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$lib timeout 300 python tools/exp_run.py --config $cfg --reps $reps --incr >> $OUT/ab.txt 2>&1
    done
  done
done
cat $OUT/ab.txt
CHECL_LIB=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so CHECL_WARP_TRACE=1 timeout 300 python tools/trace_step.py C2 4 > $OUT/warp_trace_new.txt 2>&1
grep "kernel 4" $OUT/warp_trace_new.txt | head -8
timeout 600 python tools/size_scan.py > $OUT/size_scan.txt 2>&1
cat $OUT/size_scan.txt
