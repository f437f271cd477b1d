"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck / synccheck):
every kernel shape and op of the data path on a C1-scale registry with ragged,
misaligned and zero-size buffers. Prints "sanitize ok"."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

dev = 0
sizes = [1 << 20, 0, 65536 * 3 + 17, 4097, 1, 300007]
bases = [torch.empty(s + 32, dtype=torch.uint8, device=dev) for s in sizes]
views = [b[(i % 3):(i % 3) + s] for i, (b, s) in enumerate(zip(bases, sizes))]
for i, v in enumerate(views):
    checl.debug_fill(v, 5, i)
torch.cuda.synchronize()
ctx = checl.Context()
hs = [ctx.register(v, i) for i, v in enumerate(views)]
host = [v.cpu().numpy() for v in views]
img = ctx.checkpoint(dev, epoch=1)
ctx.restore(img, dev)
d = ctx.checkpoint_device(dev, epoch=2)
ctx.restore(d, dev)
ctx.migrate(dev, dev)
for h, b in zip(hs, host):
    assert np.array_equal(ctx.tensor(h).cpu().numpy() if b.size else np.zeros(0, np.uint8), b)
# incremental + chain restore
t = ctx.tensor(hs[0])
t[12345:12346].add_(1)
torch.cuda.synchronize()
delta = ctx.checkpoint_incremental(dev, img, epoch=3)  # exact rule: seeds the shadow, diff_kernel
ctx.restore_chain([img, delta], dev)
t = ctx.tensor(hs[3])
t[100:101].add_(1)  # (a misaligned buffer in the original registry: byte path of diff_kernel before the restore)
torch.cuda.synchronize()
delta2 = ctx.checkpoint_incremental(dev, delta, epoch=5)  # shadow follows the chain
delta3 = ctx.checkpoint_incremental(dev, img, epoch=6, rule=checl.DIRTY_CRC)
for _ in range(3):  # restore fast path (cached layout, chunk-list key, in-place rebinding)
    ctx.checkpoint(dev, epoch=7, into=d)
    ctx.restore(d, dev)
ctx.set_staging(196608, 2)
img2 = ctx.checkpoint(dev, epoch=4)
ctx.restore(img2, dev)
ctx.close()
# a CRC table of >= 128 KB: the meta CRC runs on the GPU (meta_crc_kernel)
ctx = checl.Context()
big = torch.empty(40000 * 40, dtype=torch.uint8, device=dev)
checl.debug_fill(big, 9, 0)
torch.cuda.synchronize()
for i in range(40000):
    ctx.register(big[i * 40:i * 40 + 33])
d = ctx.checkpoint_device(dev, epoch=8)
ctx.restore(d, dev)
d.free()
ctx.close()
print("sanitize ok")
