"""Diagnostics: first-use cost of device allocations through PyTorch's caching allocator
(the context's default allocator) against cudaMalloc, for 80 x 64 MiB blocks."""
import time

import torch

torch.cuda.init()
torch.empty(1, device=0)
for rep in range(3):
    t0 = time.perf_counter()
    ps = [torch.cuda.caching_allocator_alloc(64 << 20, 0, 0) for _ in range(80)]
    t1 = time.perf_counter()
    for p in ps:
        torch.cuda.caching_allocator_delete(p)
    print(f"rep {rep}: torch caching_allocator_alloc 80 x 64 MiB {1e3 * (t1 - t0):.1f} ms", flush=True)
    torch.cuda.empty_cache()
t0 = time.perf_counter()
ts = [torch.empty(64 << 20, dtype=torch.uint8, device=0) for _ in range(80)]
torch.cuda.synchronize()
print(f"torch.empty 80 x 64 MiB after empty_cache {1e3 * (time.perf_counter() - t0):.1f} ms")
