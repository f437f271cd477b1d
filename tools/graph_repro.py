import sys, os
sys.path.insert(0, os.getcwd())
import torch, synth
from paper_conf_ipps_takizawakskk11_b200 import checl
w = synth.c2_sdk_mix()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
torch.cuda.synchronize()
ctx = checl.Context()
hs = [ctx.register(t) for t in ts]
img = ctx.checkpoint_device(0)
print("first ok", flush=True)
for i in range(3):
    ctx.checkpoint(0, epoch=i, into=img)
    print("into ok", i, flush=True)
    ctx.restore(img, 0)
    print("restore ok", i, flush=True)
