"""Time pack / verify kernels (device-resident image) for one library variant.
CHECL_LIB=<path> python tools/exp_run.py [--config C2] [--reps 10]"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--kind", type=int, default=0)
ap.add_argument("--incr", action="store_true", help="also time the CRC-rule incremental pass (nothing dirty)")
ap.add_argument("--mib", type=int, default=0, help="one buffer of this many MiB instead of a config")
a = ap.parse_args()
if a.mib:
    sizes, seed, streams = [a.mib << 20], 1, [0]
else:
    w = synth.CONFIGS[a.config]()
    sizes, seed, streams = [b.size for b in w.buffers], w.seed, [b.stream for b in w.buffers]
ts = [torch.empty(n, dtype=torch.uint8, device=0) for n in sizes]
for t, st in zip(ts, streams):
    checl.debug_fill(t, seed, st, a.kind)
torch.cuda.synchronize()
ctx = checl.Context()
hs = [ctx.register(t) for t in ts]
img = ctx.checkpoint_device(0)
pk, vf = [], []
for i in range(a.reps + 2):
    ctx.checkpoint(0, epoch=i, into=img)
    tp = ctx.last_timing()["kernel_ms"]
    try:
        ctx.restore(img, 0)
    except checl.CheclError:
        pass  # CHECL_EXP_PACK_OP variants write no valid image; the verify kernel still ran
    tv = ctx.last_timing()["kernel_ms"]
    if i >= 2:
        pk.append(tp)
        vf.append(tv)
S = sum(sizes)
p, v = statistics.median(pk), statistics.median(vf)
if a.incr:
    base = ctx.checkpoint(0, epoch=0)
    ci = []
    for i in range(a.reps + 2):
        d = ctx.checkpoint_incremental(0, base, epoch=i + 1, rule=checl.DIRTY_CRC)
        if i >= 2:
            ci.append(ctx.last_timing()["kernel_ms"])
        d.free()
    c = statistics.median(ci)
    print(f"  crc-rule incremental kernels {c*1e3:.1f} us ({S/c/1e6:.0f} GB/s read)")
print(f"{os.path.basename(os.path.dirname(os.environ.get('CHECL_LIB', 'default/x')))} op={os.environ.get('CHECL_EXP_PACK_OP', 0)} {a.config if not a.mib else str(a.mib) + 'MiB'}: pack {p*1e3:.1f} us "
      f"({2*S/p/1e6:.0f} GB/s 2S), verify {v*1e3:.1f} us ({2*S/v/1e6:.0f} GB/s 2S)")
