"""Minimal driver for ncu: C2 (or --config) device-resident checkpoint + restore,
`--reps` times. Used as the <cmd> of `ncu --set full -k regex:snapshot_kernel`."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--kind", type=int, default=0)
ap.add_argument("--host", action="store_true", help="pinned host image (staged pipeline)")
ap.add_argument("--flush", action="store_true", help="write 256 MB (2x L2) before every rep, like bench.py")
ap.add_argument("--verbose", action="store_true", help="kernel ms of every checkpoint / restore")
a = ap.parse_args()
w = synth.CONFIGS[a.config]()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers):
    checl.debug_fill(t, w.seed, b.stream, a.kind)
torch.cuda.synchronize()
ctx = checl.Context()
hs = [ctx.register(t) for t in ts]
img = ctx.checkpoint(0) if a.host else ctx.checkpoint_device(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=0) if a.flush else None
for i in range(a.reps):
    if flush is not None:
        flush.fill_(i & 0xFF)
    ctx.checkpoint(0, epoch=i, into=img)
    tc = ctx.last_timing()
    ctx.restore(img, 0)
    tr = ctx.last_timing()
    if a.verbose:
        print(f"rep {i}: pack {tc['kernel_ms'] * 1e3:.1f} us  verify {tr['kernel_ms'] * 1e3:.1f} us")
print(ctx.last_timing())
