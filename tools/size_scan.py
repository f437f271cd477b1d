"""Pack / verify kernel time vs payload size (one buffer), device-resident image:
separates per-launch fixed cost from the streaming rate. Prints one line per size,
beside torch's own device copy (b.copy_(a), the op MEASURED_PEAKS.json's hbm_gbs is
taken with, at 2 GiB) of the same size, timed the same way (CUDA events around one
launch, median of 6 after 2): the size-matched copy roofline."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402


def copy_us(n):
    a = torch.empty(n, dtype=torch.uint8, device=0)
    b = torch.empty_like(a)
    a.fill_(1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(8):
        torch.cuda.synchronize()
        e0.record()
        b.copy_(a)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    del a, b
    return statistics.median(ts[2:])


for mb in [int(x) for x in (sys.argv[1:] or ["16", "64", "128", "256", "442", "512", "1024", "2048", "4096"])]:
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
    img.free()
    ctx.close()
    del t
    torch.cuda.empty_cache()
    c = copy_us(n)
    torch.cuda.empty_cache()
    print(f"{mb:6d} MiB  pack {p*1e3:9.1f} us {2*n/p/1e6:7.0f} GB/s   verify {v*1e3:9.1f} us {2*n/v/1e6:7.0f} GB/s"
          f"   torch copy_ {c:9.1f} us {2*n/c/1e3:7.0f} GB/s   pack/copy_ {c/(p*1e3):.3f}", flush=True)
