"""Pack / verify kernel time vs payload size (one buffer), device-resident image:
separates per-launch fixed cost from the streaming rate. Prints one line per size."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

for mb in [int(x) for x in (sys.argv[1:] or ["16", "64", "128", "256", "512", "1024", "2048", "4096"])]:
    n = mb << 20
    t = torch.empty(n, dtype=torch.uint8, device=0)
    checl.debug_fill(t, 1, 0)
    ctx = checl.Context()
    ctx.register(t)
    img = ctx.checkpoint_device(0)
    pk, vf = [], []
    for i in range(8):
        ctx.checkpoint(0, epoch=i, into=img)
        pk.append(ctx.last_timing()["kernel_ms"])
        ctx.restore(img, 0)
        vf.append(ctx.last_timing()["kernel_ms"])
    p, v = statistics.median(pk[2:]), statistics.median(vf[2:])
    print(f"{mb:6d} MiB  pack {p*1e3:9.1f} us {2*n/p/1e6:7.0f} GB/s   verify {v*1e3:9.1f} us {2*n/v/1e6:7.0f} GB/s")
    img.free()
    ctx.close()
    del t
    torch.cuda.empty_cache()
