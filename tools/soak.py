"""Soak: many checkpoint / restore / migrate / incremental calls on C2 with the device
memory the allocator holds, the process's resident host memory and the library's
per-call timing sampled along the way; a leak shows as growth. Prints one line per
sample and a final JSON verdict."""
import json
import os
import resource
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

w = synth.c2_sdk_mix()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers):
    checl.debug_fill(t, w.seed, b.stream)
torch.cuda.synchronize()
ctx = checl.Context()
hs = [ctx.register(t) for t in ts]
dimg = ctx.checkpoint_device(0, epoch=0)
himg = ctx.checkpoint(0, epoch=0)


def rss_mb():
    with open("/proc/self/statm") as f:
        return int(f.read().split()[1]) * os.sysconf("SC_PAGE_SIZE") / 2**20


samples = []
t0 = time.time()
for it in range(2001):
    ctx.checkpoint(0, epoch=it, into=dimg)
    ctx.restore(dimg, 0)
    if it % 10 == 0:
        ctx.checkpoint(0, epoch=it, into=himg)
        ctx.restore(himg, 0)
        ctx.migrate(0, 0)
        d = ctx.checkpoint_incremental(0, himg, epoch=it + 1)
        d.free()
        tmp = ctx.checkpoint(0, epoch=it)  # a new image each time (pooled pinned memory)
        tmp.free()
    if it % 250 == 0:
        torch.cuda.synchronize()
        s = {"it": it, "t_s": round(time.time() - t0, 1), "held_MiB": torch.cuda.memory_allocated(0) / 2**20,
             "rss_MiB": round(rss_mb(), 1), "n_live": ctx.count(0)[0]}
        samples.append(s)
        print(s, flush=True)
grow_dev = samples[-1]["held_MiB"] - samples[1]["held_MiB"]
grow_rss = samples[-1]["rss_MiB"] - samples[1]["rss_MiB"]
print(json.dumps({"device_growth_MiB": grow_dev, "rss_growth_MiB": grow_rss, "samples": len(samples)}))
ctx.close()
