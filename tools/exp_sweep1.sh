python -c "import __graft_entry__ as g; g.build()" > /dev/null
for cfg in C2 C3; do
for lib in default exp_libs/w8 exp_libs/w12; do
  for op in 0 2 4; do
    if [ $lib = default ]; then L=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; else L=$PWD/$lib/libchecl.so; fi
    CHECL_LIB=$L CHECL_EXP_PACK_OP=$op timeout 120 python tools/exp_run.py --config $cfg --reps 8 2>&1 | tail -1
  done
done
done
