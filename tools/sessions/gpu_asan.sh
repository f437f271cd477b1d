#!/bin/bash
# Host-side AddressSanitizer pass: the library's host code built with -fsanitize=address
# (exp_libs/asan), preloaded into the GPU tests. Kernels are unchanged. (The two-rank
# coordination tests are left out: their spawned ranks abort in ASan's __cxa_throw
# interceptor when torch raises inside them.)
set -u
OUT=gpurun_out/${1:-asan}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
export ASAN_OPTIONS=protect_shadow_gap=0:detect_leaks=0:halt_on_error=1:log_path=$PWD/$OUT/asan
export CHECL_LIB=$PWD/exp_libs/asan/libchecl.so
LD_PRELOAD=$(gcc -print-file-name=libasan.so) timeout 2400 python -m pytest tests -m gpu -q \
  --deselect tests/test_abi.py::test_missing_library_fails_loudly --deselect tests/test_gpu_coordination.py --timeout 600 -p no:cacheprovider > $OUT/pytest.log 2>&1
echo "rc=$?" >> $OUT/pytest.log
tail -5 $OUT/pytest.log
ls $OUT
# real reports vs the spawned-child __cxa_throw aborts
grep -l "ERROR: AddressSanitizer" $OUT/asan.* 2>/dev/null | sed 's/^/REPORT: /'
grep -L "ERROR: AddressSanitizer" $OUT/asan.* 2>/dev/null | xargs -r grep -l "real___cxa_throw" | wc -l | sed 's/^/cxa_throw aborts in children: /'
