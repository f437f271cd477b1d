"""Cold vs warm host-image costs on C3 (5.35 GB): a checkpoint into a new pinned image
with the pinned pool empty (the library must pin 5.35 GB), the same with the pool
holding a freed image, and reading the image file back cold and warm. Prints JSON.

    python tools/cold_pin.py [--dir DIR]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--dir", default=os.getcwd())
ap.add_argument("--config", default="C3")
a = ap.parse_args()
w = synth.CONFIGS[a.config]()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers):
    checl.debug_fill(t, w.seed, b.stream)
torch.cuda.synchronize()
ctx = checl.Context()
for t in ts:
    ctx.register(t)
warm = ctx.checkpoint(0, epoch=0)  # (plan, staging, tables)
warm.free()


def timed(fn):
    t0 = time.perf_counter()
    r = fn()
    return time.perf_counter() - t0, r


out = {"workload": w.name, "bytes": w.total_bytes}
ctx.trim()
out["checkpoint_new_image_cold_s"], img = timed(lambda: ctx.checkpoint(0, epoch=1))
img.free()
out["checkpoint_new_image_pooled_s"], img = timed(lambda: ctx.checkpoint(0, epoch=2))
out["checkpoint_into_s"], _ = timed(lambda: ctx.checkpoint(0, epoch=3, into=img))
path = os.path.join(a.dir, f"cold_pin_{os.getpid()}.img")
img.write(path, direct=True, sync=True)
img.free()
ctx.trim()
out["read_cold_s"], back = timed(lambda: checl.Image.read(path))
out["restore_from_read_s"], _ = timed(lambda: ctx.restore(back, 0))
back.free()
out["read_pooled_s"], back = timed(lambda: checl.Image.read(path))
back.free()
os.unlink(path)
out["pin_GBs_cold"] = w.total_bytes / out["checkpoint_new_image_cold_s"] / 1e9
print(json.dumps(out))
ctx.close()
