# kernel 3 vs kernel 4 (defaults) on C1/C2/C3 + single-buffer size scan
mkdir -p gpurun_out/ab
for c in C1 C2 C3; do python tools/exp_kernels.py --config $c --kernels 3 4 --reps 8 >> gpurun_out/ab/ab.txt 2>&1; done
for k in 3 4; do echo "kernel $k" >> gpurun_out/ab/scan.txt; CHECL_KERNEL=$k python tools/size_scan.py 16 64 256 1024 4096 >> gpurun_out/ab/scan.txt 2>&1; done
