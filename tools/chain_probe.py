"""Diagnostics: where the first restores of C3 spend their time (allocator="torch" vs
"cuda"), and the raw cost of the caching allocator with C3's 10 000 tensors live."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

w = synth.c3_handle_stress()
ts = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
for t, b in zip(ts, w.buffers):
    checl.debug_fill(t, w.seed, b.stream)
torch.cuda.synchronize()
for rep in range(2):
    t0 = time.perf_counter()
    ps = [torch.cuda.caching_allocator_alloc(64 << 20, 0, 0) for _ in range(80)]
    t1 = time.perf_counter()
    for p in ps:
        torch.cuda.caching_allocator_delete(p)
    print(f"raw caching_allocator_alloc 80 x 64 MiB with C3 live, rep {rep}: {1e3 * (t1 - t0):.1f} ms", flush=True)
for alloc in ("torch", "cuda"):
    ctx = checl.Context(allocator=alloc)
    hs = [ctx.register(t) for t in ts]
    f2 = ctx.checkpoint(0, epoch=100)
    for i in range(3):
        t0 = time.perf_counter()
        ctx.restore(f2, 0)
        t1 = time.perf_counter()
        tm = ctx.last_timing()
        print(alloc, "restore", i, round((t1 - t0) * 1e3, 1), "alloc_ms", round(tm["alloc_ms"], 2), flush=True)
    f2.free()
    ctx.close()
    torch.cuda.empty_cache()
