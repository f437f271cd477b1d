# usage: bash tools/sessions/exp_sweep2.sh "<libs>" "<configs>" "<ops>" [parity-lib...]
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for lib in $1; do
for cfg in $2; do
  for op in $3; do
    if [ $lib = default ]; then L=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; else L=$PWD/exp_libs/$lib/libchecl.so; fi
    CHECL_LIB=$L CHECL_EXP_PACK_OP=$op timeout 120 python tools/exp_run.py --config $cfg --reps 8 2>&1 | tail -1 | sed "s/^/$lib /"
  done
done
done
shift 3
for lib in "$@"; do
  if [ $lib = default ]; then L=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; else L=$PWD/exp_libs/$lib/libchecl.so; fi
  CHECL_LIB=$L timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_incremental.py -x -q 2>&1 | tail -1 | sed "s/^/parity $lib: /"
done
