"""Diagnostics: device memory around migrate / restore / release (mem_get_info and
torch's allocator counters at each step)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402
from tests.gpu_util import make_set  # noqa: E402

MiB = 1 << 20
print("PYTORCH_CUDA_ALLOC_CONF", os.environ.get("PYTORCH_CUDA_ALLOC_CONF"))


def show(tag):
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    f, t = torch.cuda.mem_get_info(0)
    print(f"{tag:28s} used {(t - f) / MiB:9.1f} MiB  torch reserved {torch.cuda.memory_reserved(0) / MiB:9.1f} "
          f"allocated {torch.cuda.memory_allocated(0) / MiB:9.1f}", flush=True)


show("start")
sizes = [64 * MiB + 5, 96 * MiB, 1 * MiB + 3, 64 * MiB]
ctx = checl.Context()
ds = make_set(ctx, sizes, seed=31)
show("after make_set")
p = ctx.checkpoint_device(0, epoch=0)
show("after checkpoint_device")
p.free()
show("after free")
ctx.migrate(0, 0)
show("after migrate 1")
ctx.migrate(0, 0)
show("after migrate 2")
ctx.trim()
show("after trim")
for h in ds.handles:
    ctx.release(h)
show("after release")
ctx.trim()
show("after trim 2")
ctx.close()
show("after close")
