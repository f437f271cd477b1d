"""Live A/B of kernel shapes on one workload: one context per CHECL_KERNEL value
(read when a context first touches the device), checkpoint_into a device image +
restore, interleaved; prints the median pack / verify kernel us (library events).
usage: python tools/exp_kernels.py --config C2 --kernels 3 4 --reps 20 [--flush]"""
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
ap.add_argument("--kernels", nargs="+", default=["3", "4"])
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--flush", action="store_true")
a = ap.parse_args()
w = synth.CONFIGS[a.config]()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers):
    checl.debug_fill(t, w.seed, b.stream)
torch.cuda.synchronize()
runs = {}
for k in a.kernels:
    os.environ["CHECL_KERNEL"] = k
    ctx = checl.Context()
    for t in ts:
        ctx.register(t)
    img = ctx.checkpoint_device(0)
    runs[k] = (ctx, img, [], [])
flush = torch.empty(256 << 20, dtype=torch.uint8, device=0) if a.flush else None
for i in range(a.reps):
    for k, (ctx, img, pk, vf) in runs.items():
        if flush is not None:
            flush.fill_(i & 0xFF)
        ctx.checkpoint(0, epoch=i, into=img)
        pk.append(ctx.last_timing()["kernel_ms"] * 1e3)
        ctx.restore(img, 0)
        vf.append(ctx.last_timing()["kernel_ms"] * 1e3)
S = sum(b.size for b in w.buffers)
for k, (ctx, img, pk, vf) in runs.items():
    p, v = statistics.median(pk[2:]), statistics.median(vf[2:])
    print(f"{a.config} kernel {k}: pack {p:8.1f} us ({2 * S / p / 1e3:6.0f} GB/s)  verify {v:8.1f} us ({2 * S / v / 1e3:6.0f} GB/s)")
