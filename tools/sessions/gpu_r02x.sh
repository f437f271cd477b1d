#!/bin/bash
# Fuzz on the round's final code: 400 default-dispatch cases, 150 each with every launch
# forced to kernel 1 (snapshot) and kernel 2 (sweep) (their table copies now overlap the
# first loads), and 200 registry/snapshot call sequences.
set -u
OUT=gpurun_out/${1:-r02x}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
CHECL_FUZZ_CASES=400 timeout 900 python -m pytest tests/test_gpu_fuzz.py -q > $OUT/fuzz400.log 2>&1; tail -1 $OUT/fuzz400.log
CHECL_KERNEL=1 CHECL_FUZZ_CASES=150 timeout 900 python -m pytest tests/test_gpu_fuzz.py -q > $OUT/fuzz150_k1.log 2>&1; tail -1 $OUT/fuzz150_k1.log
CHECL_KERNEL=2 CHECL_FUZZ_CASES=150 timeout 900 python -m pytest tests/test_gpu_fuzz.py -q > $OUT/fuzz150_k2.log 2>&1; tail -1 $OUT/fuzz150_k2.log
CHECL_REG_FUZZ_CASES=200 timeout 1200 python -m pytest tests/test_gpu_registry_fuzz.py -q > $OUT/regfuzz200.log 2>&1; tail -1 $OUT/regfuzz200.log
