#!/bin/bash
# Multi-rank bench path after this round's bench changes: two ranks sharing the GPU over
# gloo (timings meaningless), C3 coordinated every step, C5 both routes, reference arm.
set -u
O=gpurun_out/${1:-r02u}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
export CHECL_BENCH_DIST_BACKEND=gloo
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu-baseline > $O/torchrun2_c3.json 2> $O/torchrun2_c3.err; echo "c3 rc=$?"
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 2 --config C5 --steps 5 --warmup 3 > $O/torchrun2_c5.json 2> $O/torchrun2_c5.err; echo "c5 rc=$?"
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29536 bench.py --gpus 2 --impl reference --steps 2 --warmup 3 > $O/torchrun2_ref.json 2> $O/torchrun2_ref.err; echo "ref rc=$?"
for f in $O/torchrun2_*.json; do echo "== $f"; head -c 600 $f; echo; done
