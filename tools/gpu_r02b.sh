#!/bin/bash
# incremental (both rules) + memory tests, memory diagnostics, C2 segment A/B
set -u
O=gpurun_out/${1:-r02b}
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_incremental.py tests/test_gpu_memory.py tests/test_gpu_coordination.py -q > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -15 $O/pytest.log
timeout 300 python tools/mem_diag.py > $O/mem_diag.txt 2>&1; cat $O/mem_diag.txt
for rule in bytes crc; do for d in 0.01 0.1; do
  timeout 300 python bench.py --mode incremental --dirty $d --rule $rule > $O/inc_${rule}_$d.json 2> $O/inc_${rule}_$d.err
  python -c "import json;d=json.load(open('$O/inc_${rule}_$d.json'));print('$rule $d', 'ms %.3f full %.3f speedup %.1f kernel %.3f verified %s present %d' % (d['ms_per_step'], d['full_checkpoint_ms'], d['speedup_vs_full'], d['kernel_ms_per_step'], d['verified'], d['present_chunks_per_step']))" 2>&1 | tail -1
done; done
for rep in 1 2; do for seg in default 0; do
  if [ $seg = default ]; then E=""; else E="CHECL_SEGMENT_BYTES=0"; fi
  env $E timeout 300 python bench.py --config C2 --no-cpu-baseline --no-extras --no-e2e > $O/c2_seg${seg}_$rep.json 2>/dev/null
  python -c "import json;d=json.load(open('$O/c2_seg${seg}_$rep.json'));r=d['roofline'];print('C2 seg=$seg', 'value %.1f step %.4f pack %.1f verify %.1f' % (d['value'], d['ms_per_step'], r['pack_ms']*1e3, r['verify_ms']*1e3))" 2>&1 | tail -1
done; done
