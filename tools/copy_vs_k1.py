"""K1 / K2 beside torch's copy_ of the same payload size on one workload (device image),
for an ncu launch list: run under `ncu --metrics gpu__time_duration.sum,...` to compare
the kernels' own durations, and without ncu for CUDA-event spans.
usage: python tools/copy_vs_k1.py [config] [reps]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
w = synth.CONFIGS[cfg]()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers):
    checl.debug_fill(t, w.seed, b.stream)
S = w.total_bytes
a = torch.empty(S, dtype=torch.uint8, device=0)
b = torch.empty_like(a)
a.fill_(3)
ctx = checl.Context()
for t in ts:
    ctx.register(t)
img = ctx.checkpoint_device(0)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
pk, vf, cp = [], [], []
for i in range(reps + 1):
    ctx.checkpoint(0, epoch=i, into=img)
    pk.append(ctx.last_timing()["kernel_ms"] * 1e3)
    ctx.restore(img, 0)
    vf.append(ctx.last_timing()["kernel_ms"] * 1e3)
    torch.cuda.synchronize()
    e0.record()
    b.copy_(a)
    e1.record()
    torch.cuda.synchronize()
    cp.append(e0.elapsed_time(e1) * 1e3)
p, v, c = (statistics.median(x[1:]) for x in (pk, vf, cp))
print(f"{cfg} S={S}: pack {p:.1f} us, verify {v:.1f} us, torch copy_ {c:.1f} us (events, median of {reps})")
