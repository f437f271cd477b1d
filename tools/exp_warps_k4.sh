# Warps per CTA for kernel 4 (exp_libs/w8, w9, w10), C2 and C3, interleaved passes.
O=gpurun_out/wk4
mkdir -p $O
for pass in 1 2 3; do
 for w in w8 w9 w10; do
  echo "$w $(CHECL_LIB=$PWD/exp_libs/$w/libchecl.so timeout 120 python tools/exp_kernels.py --config C2 --kernels 4 --reps 12 2>&1 | tail -1)" >> $O/sweep.txt
 done
done
for w in w8 w10; do
  echo "$w $(CHECL_LIB=$PWD/exp_libs/$w/libchecl.so timeout 300 python tools/exp_kernels.py --config C3 --kernels 4 --reps 5 2>&1 | tail -1)" >> $O/sweep.txt
done
cat $O/sweep.txt
