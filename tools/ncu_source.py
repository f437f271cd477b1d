"""Top SASS lines by warp-stall samples from an .ncu-rep source page."""
import csv
import io
import subprocess
import sys

rep, which = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "0"
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
blocks, cur = [], None
for row in csv.reader(io.StringIO(out)):
    if row and row[0] == "Kernel Name":
        cur = {"name": row[1], "rows": []}
        blocks.append(cur)
    elif cur is not None:
        cur["rows"].append(row)
for b in blocks:
    if f"<(bool){which}>" not in b["name"] and which not in b["name"]:
        continue
    hdr, rows = b["rows"][0], b["rows"][1:]
    si = hdr.index("Warp Stall Sampling (All Samples)")
    stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") or "Stall" in h and i > si + 2]
    tot = sum(int(r[si] or 0) for r in rows)
    print(b["name"], "total samples", tot)
    rows.sort(key=lambda r: -int(r[si] or 0))
    for r in rows[:top]:
        print(f"{int(r[si]):7d} {100*int(r[si])/tot:5.1f}%  {r[1].strip()[:70]}")
    # aggregate by opcode
    agg = {}
    for r in rows:
        op = r[1].strip().split()[0] if r[1].strip() else "?"
        if op.startswith("@"):
            op = r[1].strip().split()[1]
        op = op.split(".")[0]
        agg[op] = agg.get(op, 0) + int(r[si] or 0)
    print("by opcode:", ", ".join(f"{k}={100*v/tot:.1f}%" for k, v in sorted(agg.items(), key=lambda x: -x[1])[:14]))
