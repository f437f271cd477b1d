#!/bin/bash
# Sweep kernel (C1-sized launches): table copy overlapped with the first unit's loads.
# Kernel-shape + parity tests, then pack / verify against the previous commit
# (exp_libs/prev) on C1 (and one 6 MiB buffer), three passes; the C1 bench line.
set -u
OUT=gpurun_out/${1:-r02w}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_incremental.py tests/test_gpu_modes.py -x -q > $OUT/pytest.log 2>&1
tail -2 $OUT/pytest.log
NEW=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so
OLD=$PWD/exp_libs/prev/libchecl.so
for pass in 1 2 3; do
  for args in "--config C1 --reps 60" "--mib 6 --reps 60"; do
    for v in old new; do
      if [ $v = new ]; then lib=$NEW; else lib=$OLD; fi
      echo -n "$v " >> $OUT/ab.txt
      CHECL_LIB=$lib timeout 300 python tools/exp_run.py $args >> $OUT/ab.txt 2>&1
    done
  done
done
cat $OUT/ab.txt
for v in old new; do
  if [ $v = new ]; then lib=$NEW; else lib=$OLD; fi
  CHECL_LIB=$lib timeout 600 python bench.py --config C1 --no-cpu-baseline --no-extras > $OUT/bench_c1_$v.json 2> $OUT/bench_c1_$v.err
  python -c "import json;d=json.load(open('$OUT/bench_c1_$v.json'));print('$v', d['value'], d['ms_per_step'], d['roofline']['pack_ms'], d['roofline']['verify_ms'], d['e2e']['value'])"
done
