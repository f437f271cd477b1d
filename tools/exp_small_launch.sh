#!/bin/bash
# Small-launch kernel choice: pack / verify kernel time vs payload size (one buffer,
# HBM image) with the sweep kernel (2), the balanced kernel (3) and the default.
mkdir -p gpurun_out/small
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/small/build.log 2>&1
for k in 0 2 3; do
  echo "== CHECL_KERNEL=$k"
  CHECL_KERNEL=$k timeout 300 python tools/size_scan.py 1 2 3 4 6 8 12 16 24 32
done 2>&1 | tee gpurun_out/small/scan.txt
