# kernel-shape comparison: default vs variant libs under CHECL_KERNEL=1/3
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for lib in default $1; do
  if [ $lib = default ]; then L=$PWD/paper_conf_ipps_takizawakskk11_b200/libchecl.so; else L=$PWD/exp_libs/$lib/libchecl.so; fi
  for k in 1 3; do for cfg in C2 C3; do
    CHECL_LIB=$L CHECL_KERNEL=$k timeout 120 python tools/exp_run.py --config $cfg --reps 8 2>&1 | tail -1 | sed "s/^/$lib k=$k /"
  done; done
done
