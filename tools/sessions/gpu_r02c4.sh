python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
mkdir -p gpurun_out/r02c4
S=$(date +%s)
timeout 1500 python bench.py --config C4 --no-cpu-baseline > gpurun_out/r02c4/bench_c4.json 2> gpurun_out/r02c4/bench_c4.err; echo rc=$? elapsed=$(( $(date +%s) - S ))s
python -c "import json;d=json.load(open('gpurun_out/r02c4/bench_c4.json'));print(d['value'], d['roofline']['frac'], d['roofline'].get('copy_same_size'), d['e2e']['value'], d['e2e'].get('drain_frac_of_pcie'), d['e2e'].get('fill_frac_of_pcie'), d['clocks'])"
