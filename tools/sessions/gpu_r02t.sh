#!/bin/bash
# Column-register rounds for the CRC-only ops (CHECL_CRC_LDG): parity (kernel shapes,
# parity, fuzz, incremental), then the CRC-rule pass / pack / verify against the same
# code built with -DCHECL_CRC_LDG=0 (exp_libs/ldg0), C2 and C3, three passes; ncu of
# the CRC-only kernel on C3 both ways.
set -u
OUT=gpurun_out/${1:-r02t}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_incremental.py -x -q > $OUT/pytest.log 2>&1
tail -3 $OUT/pytest.log
NEW=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so
OLD=$PWD/exp_libs/ldg0/libchecl.so
for pass in 1 2 3; do
  for cfg in C2 C3; do
    reps=30; [ $cfg = C3 ] && reps=8
    for v in old new; do
      if [ $v = new ]; then lib=$NEW; else lib=$OLD; fi
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$lib timeout 300 python tools/exp_run.py --config $cfg --reps $reps --incr >> $OUT/ab.txt 2>&1
    done
  done
done
cat $OUT/ab.txt
for v in old new; do
  if [ $v = new ]; then lib=$NEW; else lib=$OLD; fi
  CHECL_LIB=$lib timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"tma_kernel<2" -c 1 -o /tmp/crc_$v -f python tools/exp_run.py --config C3 --reps 1 --incr > $OUT/ncu_$v.log 2>&1
  python tools/ncu_summary.py /tmp/crc_$v.ncu-rep > $OUT/crc_summary_$v.txt 2>&1
  ncu -i /tmp/crc_$v.ncu-rep --page raw --csv > $OUT/crc_raw_$v.csv 2>&1
done
head -40 $OUT/crc_summary_new.txt
