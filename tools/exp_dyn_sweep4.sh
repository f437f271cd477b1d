# Re-sweep of the kernel-4 work split on the current code (graph launches, one-probe
# find_chunk): static share (permille) x dynamic block (rounds), C2, two passes.
O=gpurun_out/dyn4
mkdir -p $O
for pass in 1 2; do
for sp in 650 750 850 900; do
 for b in 4 8 12 16; do
  echo "sp=$sp b=$b $(CHECL_STATIC_PERMILLE=$sp CHECL_DYN_BLOCK=$b timeout 120 python tools/exp_kernels.py --config C2 --kernels 4 --reps 12 2>&1 | tail -1)" >> $O/sweep.txt
 done
done
done
cat $O/sweep.txt
