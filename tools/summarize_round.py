"""Write the judged summaries of one GPU session into profiles/<round>/ and
profiles/traffic.json (per-launch DRAM bytes of K1/K2 from the ncu --set full capture).
usage: python tools/summarize_round.py <gpurun_out/tag> <profiles/rNN> [config of prof.ncu-rep, default C3]"""
import csv
import io
import json
import os
import re
import shutil
import sys
from collections import defaultdict

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summary  # noqa: E402

src, dst = sys.argv[1], sys.argv[2]
CFG = sys.argv[3] if len(sys.argv) > 3 else "C3"
os.makedirs(dst, exist_ok=True)
import glob  # noqa: E402
for f in sorted(glob.glob(os.path.join(src, "bench*.json"))) + [
        os.path.join(src, f) for f in ("pytest_gpu.log", "smoke.log", "nvsmi.txt", "trace.log", "trace_c3.log", "sanitizer.txt")]:
    if os.path.exists(f):
        shutil.copy(f, os.path.join(dst, os.path.basename(f)))
lines = []
lc = os.path.join(src, "launches.csv")
if os.path.exists(lc):
    shutil.copy(lc, os.path.join(dst, "launches.csv"))
    rows = list(csv.reader(open(lc)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    agg = defaultdict(list)
    for r in rows[hi + 1:]:
        if len(r) > h.index("Metric Value"):
            agg[r[h.index("Kernel Name")].split("(")[0]].append(float(r[h.index("Metric Value")].replace(",", "")))
    tot = sum(sum(v) for v in agg.values())
    lines += ["## Launch list (ncu gpu__time_duration.sum, --clock-control none; cold, serialised)", "",
              "| kernel | launches | mean us | share of kernel time |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
        lines.append(f"| `{k}` | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {100 * sum(v) / tot:.1f}% |")
    lines.append("")
rep = os.path.join(src, "prof.ncu-rep")
traffic = {}
if os.path.exists(rep):
    lines += [f"## ncu --set full ({CFG}, device-resident image; tools/profile_step.py)", ""]
    for d in summary(rep):
        name = d.pop("kernel")
        st = d.pop("stalls_per_issue")
        lines.append(f"### `{name}`")
        lines.append("")
        for k, (v, u) in d.items():
            lines.append(f"- {k}: {v} {u}")
        lines.append("- stalls per issue: " + ", ".join(f"{k} {v:.2f}" for k, v in st.items()))
        lines.append("")
        rd = float(d["dram__bytes_read.sum"][0]) * (1e6 if "Mbyte" in d["dram__bytes_read.sum"][1] else 1e9 if "Gbyte" in d["dram__bytes_read.sum"][1] else 1)
        wr = float(d["dram__bytes_write.sum"][0]) * (1e6 if "Mbyte" in d["dram__bytes_write.sum"][1] else 1e9 if "Gbyte" in d["dram__bytes_write.sum"][1] else 1)
        # first template argument = the kOp (checl_internal.h): 0 pack (K1), 1 verify (K2)
        m = re.search(r"<\s*(\d+)", name)
        op = int(m.group(1)) if m else -1
        if op in (0, 1):
            traffic["K1" if op == 0 else "K2"] = rd + wr
if os.path.exists(os.path.join(src, "bench.json")):
    try:
        b = json.loads(open(os.path.join(src, "bench.json")).read().strip().splitlines()[-1])
        lines = [f"## bench.py ({b['config']['workload']}, N=1)", "", "```", json.dumps({k: b[k] for k in ("value", "unit", "ms_per_step", "roofline", "e2e", "clocks", "cpu_baseline", "extras") if k in b}, indent=1), "```", ""] + lines
    except Exception as e:
        lines.insert(0, f"(bench.json unreadable: {e})")
open(os.path.join(dst, "SUMMARY.md"), "w").write("# GPU session summary\n\n" + "\n".join(lines) + "\n")
if traffic:
    tp = os.path.join(os.path.dirname(dst.rstrip("/")), "traffic.json")
    cur = json.load(open(tp)) if os.path.exists(tp) else {}
    cur[CFG] = {"dram_bytes_per_launch": max(traffic.values()), "K1": traffic.get("K1"), "K2": traffic.get("K2"),
                 "source": f"{dst}/SUMMARY.md (ncu --set full dram__bytes_read.sum + dram__bytes_write.sum)"}
    json.dump(cur, open(tp, "w"), indent=1)
print(open(os.path.join(dst, "SUMMARY.md")).read()[:3000])
