# Sweep of the dynamic-tail parameters (DESIGN.md §5 "Work split"): kernel x static
# share (permille) x dynamic block (rounds), C2 (and C3) live A/B timings.
mkdir -p gpurun_out/dyn2
for k in 4; do
 for sp in 700 800 900; do
  for b in 8 16 32; do
   echo "k=$k sp=$sp b=$b $(CHECL_STATIC_PERMILLE=$sp CHECL_DYN_BLOCK=$b timeout 120 python tools/exp_kernels.py --config C2 --kernels $k --reps 10 2>&1 | tail -1)" >> gpurun_out/dyn2/sweep.txt
  done
 done
done
for sp in 1000 800 900; do
 for k in 3 4; do
  echo "k=$k sp=$sp b=16 $(CHECL_STATIC_PERMILLE=$sp CHECL_DYN_BLOCK=16 timeout 300 python tools/exp_kernels.py --config C3 --kernels $k --reps 4 2>&1 | tail -1)" >> gpurun_out/dyn2/sweep.txt
 done
done
