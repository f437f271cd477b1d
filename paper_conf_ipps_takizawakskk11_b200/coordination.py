"""Coordinated checkpoint across the ranks of one box (global snapshot).

PAPER.md L40 §IV-C: "The checkpoint files of individual computing nodes, called
local snapshots, are aggregated into a global snapshot [14]" (Open MPI's CPR). Here
each rank snapshots its own GPU's buffers independently (no data crosses ranks);
the only exchange is one 88-byte status all-reduce over the process group (NCCL over
NVLink on GPUs, gloo in CPU tests): SUM of [failures, buffers, bytes] and of the
epoch's 16-bit parts and their squares (agreement test in `agree`). The global snapshot commits iff no rank failed and every rank
checkpointed the same epoch (reading 16: a two-phase commit); otherwise
every rank frees its local image.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Callable, Optional, Tuple


@dataclass
class GlobalSnapshot:
    committed: bool
    image: object  # the local Image, or None when aborted
    failures: int
    n_buffers: int
    total_bytes: int
    epoch: int
    epochs_agree: bool


def agree(failed: bool, n_buffers: int, nbytes: int, epoch: int, group=None, device=None) -> Tuple[int, int, int, bool, int]:
    """The coordination all-reduce — ONE all-reduce (SUM) of 11 int64 per rank.
    Returns (failures, buffers, bytes, epochs_agree, epoch).

    Epoch agreement without a MAX: the 64-bit epoch is split into four 16-bit parts
    x_k and every rank contributes x_k and x_k^2; by the equality case of
    Cauchy-Schwarz, all ranks hold the same x_k iff N * sum(x_k^2) == (sum x_k)^2
    (exact: x_k < 2^16, so nothing overflows int64 for any world size < 2^31)."""
    import torch
    import torch.distributed as dist

    dev = torch.device("cuda", device) if (device is not None and dist.get_backend(group) == "nccl") else torch.device("cpu")
    e = epoch & 0xFFFFFFFFFFFFFFFF
    parts = [(e >> (16 * k)) & 0xFFFF for k in range(4)]
    s = torch.tensor([1 if failed else 0, n_buffers, nbytes] + parts + [x * x for x in parts], dtype=torch.int64, device=dev)
    dist.all_reduce(s, op=dist.ReduceOp.SUM, group=group)
    v = s.cpu().tolist()
    n = dist.get_world_size(group)
    same = all(n * v[7 + k] == v[3 + k] * v[3 + k] for k in range(4))
    agreed = sum((v[3 + k] // n) << (16 * k) for k in range(4)) if same else epoch
    return int(v[0]), int(v[1]), int(v[2]), same, int(agreed)


def coordinated(take_local: Callable[[], Tuple[object, int, int]], epoch: int, group=None,
                device: Optional[int] = None, keep=None) -> GlobalSnapshot:
    """Runs `take_local()` -> (image, n_buffers, bytes) on every rank, then the
    status all-reduce; frees the local image if the global snapshot aborts, unless it
    is `keep` (a caller-owned image reused through checl_checkpoint_into: the caller
    keeps it, and `committed` = False says its contents are not a global snapshot)."""
    img, n, b, failed = None, 0, 0, False
    try:
        img, n, b = take_local()
    except Exception:
        failed = True
    f, tn, tb, same, ep = agree(failed, n, b, epoch, group, device)
    ok = f == 0 and same
    if not ok and img is not None:
        if img is not keep:
            img.free()
        img = None
    return GlobalSnapshot(ok, img, f, tn, tb, ep, same)


class ImagePair:
    """Two reusable host images for a loop of global snapshots (double buffering).

    Each new local snapshot is written into the image that does NOT hold the last
    committed global snapshot, so an aborted vote leaves the last committed one
    intact: the rollback target of the two-phase commit (reading 16).
    `committed` is that image (None before the first commit). Neither image is
    re-pinned after its first use."""

    def __init__(self):
        self.images = [None, None]
        self.last = -1  # index of the committed image

    @property
    def committed(self):
        return self.images[self.last] if self.last >= 0 else None

    def _slot(self) -> int:
        return 0 if self.last != 0 else 1

    def take(self, ctx, device: int, stream, epoch: int):
        k = self._slot()
        if self.images[k] is None:
            self.images[k] = ctx.checkpoint(device, stream, epoch)
        else:
            ctx.checkpoint(device, stream, epoch, into=self.images[k])
        return self.images[k]

    def commit(self, img):
        self.last = self.images.index(img)

    def free(self):
        for im in self.images:
            if im is not None:
                im.free()
        self.images = [None, None]
        self.last = -1


def coordinated_checkpoint(ctx, device: int, epoch: int, group=None, stream=None, into=None,
                           on_device: bool = False) -> GlobalSnapshot:
    """Local checl_checkpoint (host image, or HBM image with on_device) + commit barrier.

    into=None: a new image; freed on abort. into=Image: written in place (no
    re-pinning) and kept on abort, but its previous contents are overwritten before
    the vote, so an abort leaves no committed snapshot to roll back to. into=ImagePair:
    double-buffered, an abort keeps the last committed snapshot intact (snap.image is
    then None and pair.committed is the previous global snapshot)."""
    pair = into if isinstance(into, ImagePair) else None

    def local():
        n, b = ctx.count(device)
        if on_device:
            return ctx.checkpoint_device(device, stream, epoch), n, b
        if pair is not None:
            return pair.take(ctx, device, stream, epoch), n, b
        return ctx.checkpoint(device, stream, epoch, into=into), n, b

    if pair is not None:
        k = pair._slot()
        target = pair.images[k]  # None: the slot's first snapshot (a new image, freed on abort)
        snap = coordinated(local, epoch, group, device, keep=target)
        if snap.committed:
            pair.commit(snap.image)
        elif target is None:
            pair.images[k] = None
        return snap
    return coordinated(local, epoch, group, device, keep=into)
