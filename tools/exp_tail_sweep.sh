# Fine-tail sweep (DESIGN.md §5 "Work split"): the last T permille of the dynamic
# rounds in blocks of b rounds; C2 and C3, kernel 4, live timings + warp trace.
O=gpurun_out/tail
mkdir -p $O
for tp in 0 200 400; do
 for b in 1 2 4; do
  if [ $tp = 0 ] && [ $b != 2 ]; then continue; fi
  echo "tail=$tp b=$b $(CHECL_TAIL_PERMILLE=$tp CHECL_TAIL_BLOCK=$b timeout 120 python tools/exp_kernels.py --config C2 --kernels 4 --reps 12 2>&1 | tail -1)" >> $O/sweep.txt
 done
done
for tp in 0 200 400; do
  echo "tail=$tp b=2 $(CHECL_TAIL_PERMILLE=$tp CHECL_TAIL_BLOCK=2 timeout 300 python tools/exp_kernels.py --config C3 --kernels 4 --reps 4 2>&1 | tail -1)" >> $O/sweep.txt
done
CHECL_TAIL_PERMILLE=400 CHECL_TAIL_BLOCK=2 CHECL_WARP_TRACE=1 python tools/profile_step.py --config C2 --reps 3 > $O/trace.txt 2>&1
