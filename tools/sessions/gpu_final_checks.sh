#!/bin/bash
# Robustness pass on the final code: compute-sanitizer (memcheck / racecheck / synccheck)
# x (default dispatch, kernel 3, kernel 4 with the dynamic tail forced), a 400-case GPU
# fuzz, and the host phase trace of C1. usage: tools/sessions/gpu_final_checks.sh <tag>
set -u
O=gpurun_out/${1:-final}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_default.log 2>&1
  CHECL_KERNEL=3 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_3.log 2>&1
  CHECL_LIB=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl_exp.so CHECL_KERNEL=4 CHECL_DYN_MIN_ROUNDS=0 CHECL_STATIC_PERMILLE=300 CHECL_DYN_BLOCK=2 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_4dyn.log 2>&1
done
for f in $O/san_*.log; do echo "== $(basename $f)"; grep -E "sanitize ok|SUMMARY" $f; done > $O/sanitizer.txt
CHECL_FUZZ_CASES=400 timeout 900 python -m pytest tests/test_gpu_fuzz.py -m gpu -q > $O/fuzz400.log 2>&1
CHECL_TRACE=1 timeout 120 python tools/trace_step.py C1 8 > $O/trace_c1.log 2>&1
cat $O/sanitizer.txt; tail -1 $O/fuzz400.log
