#!/bin/bash
# multi-rank runs on one GPU (gloo), Eq. (1) cost model, filtered launch list,
# CRC-only pass and K1 source-level ncu, the default bench line.
set -u
O=gpurun_out/${1:-r02f}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
df -h . /tmp /dev/shm > $O/df.txt 2>&1; mount | grep -E " / | /tmp | /root" >> $O/df.txt
export CHECL_BENCH_DIST_BACKEND=gloo
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu-baseline > $O/torchrun2_c3.json 2> $O/torchrun2_c3.err; echo "c3 rc=$?"
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 2 --config C5 --steps 5 --warmup 3 > $O/torchrun2_c5.json 2> $O/torchrun2_c5.err; echo "c5 rc=$?"
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29535 bench.py --gpus 2 --config C5 --c5-route copy --steps 5 --warmup 3 > $O/torchrun2_c5_copy.json 2> $O/torchrun2_c5_copy.err; echo "c5 copy rc=$?"
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29536 bench.py --gpus 2 --impl reference --steps 2 --warmup 3 > $O/torchrun2_ref.json 2> $O/torchrun2_ref.err; echo "ref rc=$?"
unset CHECL_BENCH_DIST_BACKEND
tail -c 400 $O/torchrun2_c3.json; echo; tail -c 300 $O/torchrun2_c5.json; echo
timeout 1500 python tools/cost_model.py --dir $PWD --reps 5 > $O/cost_model_disk.json 2> $O/cost_model_disk.err; echo "cost disk rc=$?"
timeout 1200 python tools/cost_model.py --dir /dev/shm --reps 5 > $O/cost_model_tmpfs.json 2> $O/cost_model_tmpfs.err; echo "cost tmpfs rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"tma_kernel|sweep_kernel|balanced_kernel|snapshot_kernel|expand_plan|build_tables" -c 200 --csv --log-file $O/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-extras > $O/launches.log 2>&1
R=/tmp/ncu_$$; mkdir -p $R
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tma_kernel<2" -c 2 -o $R/crc -f python bench.py --mode incremental --config C2 --steps 1 --warmup 1 --dirty 0.01 --rule crc > $O/ncu_crc.log 2>&1
python tools/ncu_summary.py $R/crc.ncu-rep > $O/crc_summary.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"tma_kernel<0" -s 1 -c 1 -o $R/k1 -f python tools/profile_step.py --config C2 --reps 2 > $O/ncu_k1.log 2>&1
ncu -i $R/k1.ncu-rep --page source --csv --print-source sass > $O/k1_source_sass.csv 2>&1
ncu -i $R/k1.ncu-rep --page source --csv > $O/k1_source.csv 2>&1
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
python -c "
import json;d=json.load(open('$O/bench.json'));r=d['roofline'];e=d['e2e']
print('C3 value %.1f step %.3f frac %.3f traffic %s e2e %.2f' % (d['value'], d['ms_per_step'], r['frac'], r['traffic'], e['value']))
for k,v in d['extras'].items(): print(k, v.get('value'), v.get('roofline',{}).get('frac'), v.get('error'))"
du -sh $O
