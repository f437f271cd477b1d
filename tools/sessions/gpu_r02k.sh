#!/bin/bash
# Quad-chain CRC from registers / LDS.128: parity of the default build, then A/B
# against the previous build (prev) and the CRC-from-registers variant (creg).
set -u
OUT=gpurun_out/${1:-r02k}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_kernels.py tests/test_gpu_incremental.py tests/test_gpu_fuzz.py tests/test_gpu_registry_fuzz.py tests/test_gpu_modes.py -x -q > $OUT/pytest.log 2>&1
tail -3 $OUT/pytest.log
lib() { if [ $1 = default ]; then echo $PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; else echo $PWD/exp_libs/$1/libchecl.so; fi; }
for cfg in C2 C3; do
  reps=20; [ $cfg = C3 ] && reps=6
  for pass in 1 2; do
    for v in prev default creg; do
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$(lib $v) timeout 300 python tools/exp_run.py --config $cfg --reps $reps --incr >> $OUT/ab.txt 2>&1
    done
  done
done
for pass in 1 2; do
  for v in prev default; do
    echo -n "remote $v " >> $OUT/ab.txt
    CHECL_FORCE_IMAGE_REMOTE=1 CHECL_LIB=$(lib $v) timeout 300 python tools/exp_run.py --config C2 --reps 20 >> $OUT/ab.txt 2>&1
  done
done
cat $OUT/ab.txt
