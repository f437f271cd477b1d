import sys, os
sys.path.insert(0, os.getcwd())
import torch, synth
from paper_conf_ipps_takizawakskk11_b200 import checl
w = synth.c2_sdk_mix()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers): checl.debug_fill(t, 2, b.stream)
torch.cuda.synchronize()
ctx = checl.Context()
for t in ts: ctx.register(t)
img = ctx.checkpoint_device(0)
for i in range(8):
    ctx.checkpoint(0, epoch=i, into=img)
    ctx.restore(img, 0)
