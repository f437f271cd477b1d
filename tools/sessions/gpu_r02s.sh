#!/bin/bash
# C2: K1 / K2 against torch's copy_ of the same size, events and ncu durations; the
# bench line with the same-size copy field.
set -u
OUT=gpurun_out/${1:-r02s}
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for cfg in C2 C3; do timeout 300 python tools/copy_vs_k1.py $cfg 8 >> $OUT/events.txt 2>&1; done
cat $OUT/events.txt
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__cycles_active.avg --clock-control none --csv --log-file $OUT/ncu_c2.csv python tools/copy_vs_k1.py C2 4 > $OUT/ncu_c2.log 2>&1
python - <<'PY' >> $OUT/ncu_summary.txt
import csv, collections
rows = list(csv.DictReader(l for l in open("gpurun_out/${1:-r02s}/ncu_c2.csv") if l.startswith('"')))
agg = collections.defaultdict(lambda: collections.defaultdict(list))
for r in rows:
    k = r["Kernel Name"][:60]
    try: agg[k][r["Metric Name"]].append(float(r["Metric Value"].replace(",", "")))
    except ValueError: pass
for k, m in agg.items():
    print(k, {n: round(sorted(v)[len(v)//2], 1) for n, v in m.items()}, "n=%d" % len(m["gpu__time_duration.sum"]))
PY
cat $OUT/ncu_summary.txt
timeout 600 python bench.py --config C2 --no-cpu-baseline --no-extras > $OUT/bench_c2.json 2> $OUT/bench_c2.err
python -c "import json;d=json.load(open('$OUT/bench_c2.json'));print(json.dumps(d['roofline']))"
