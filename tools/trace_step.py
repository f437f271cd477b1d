"""CHECL_TRACE=1 host phase trace of checkpoint_into + restore on a device image.
usage: CHECL_TRACE=1 python tools/trace_step.py [config] [reps] [host]  (host: pinned host image)"""
import os
import sys

sys.path.insert(0, os.getcwd())
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 8
w = synth.CONFIGS[cfg]()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers):
    checl.debug_fill(t, w.seed, b.stream)
torch.cuda.synchronize()
ctx = checl.Context()
for t in ts:
    ctx.register(t)
img = ctx.checkpoint(0) if len(sys.argv) > 3 and sys.argv[3] == "host" else ctx.checkpoint_device(0)
for i in range(reps):
    ctx.checkpoint(0, epoch=i, into=img)
    ctx.restore(img, 0)
