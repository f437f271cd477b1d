# Sweep of the dynamic-tail parameters (DESIGN.md §5 "Work split"): static share
# (permille) x dynamic block (rounds), kernel 4, C2 and C3 live timings.
O=gpurun_out/dyn3
mkdir -p $O
for sp in 650 750 850; do
 for b in 4 6 8 12; do
  echo "sp=$sp b=$b $(CHECL_STATIC_PERMILLE=$sp CHECL_DYN_BLOCK=$b timeout 120 python tools/exp_kernels.py --config C2 --kernels 4 --reps 10 2>&1 | tail -1)" >> $O/sweep.txt
 done
done
for sp in 750 850; do
 for b in 6 8; do
  echo "sp=$sp b=$b $(CHECL_STATIC_PERMILLE=$sp CHECL_DYN_BLOCK=$b timeout 300 python tools/exp_kernels.py --config C3 --kernels 4 --reps 4 2>&1 | tail -1)" >> $O/sweep.txt
 done
done
