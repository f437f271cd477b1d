"""Helpers for the -m gpu parity tests: build registries on the device with the
synth/ generator and host copies made by plain cudaMemcpy (torch .cpu())."""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Sequence

import numpy as np



@dataclass
class DevSet:
    tensors: list       # the registered views
    bases: list         # owning allocations
    handles: List[int]
    host: List[np.ndarray]
    flags: List[int]


def make_set(ctx, sizes: Sequence[int], seed: int = 1, offsets: Sequence[int] = None, kind: int = 0,
             device: int = 0, flags: Sequence[int] = None) -> DevSet:
    import torch
    from paper_conf_ipps_takizawakskk11_b200 import checl
    offsets = offsets or [0] * len(sizes)
    flags = list(flags) if flags is not None else [(0x1000 + i) for i in range(len(sizes))]
    bases, views, handles, host = [], [], [], []
    for i, (s, o) in enumerate(zip(sizes, offsets)):
        b = torch.empty(s + o + 16, dtype=torch.uint8, device=device)
        v = b[o:o + s]
        checl.debug_fill(v, seed, i, kind)
        bases.append(b)
        views.append(v)
    torch.cuda.synchronize(device)
    for v, f in zip(views, flags):
        handles.append(ctx.register(v, f))
    host = [v.cpu().numpy() for v in views]
    return DevSet(views, bases, handles, host, flags)


def oracle_entries(ds: DevSet):
    from oracle import oracle as O
    return [O.Entry(h, b, f) for h, b, f in zip(ds.handles, ds.host, ds.flags)]


def release_all(ctx, ds: DevSet):
    for h in ds.handles:
        try:
            ctx.release(h)
        except Exception:
            pass


def bound_bytes(ctx, handle: int) -> np.ndarray:
    ptr, nb, dev = ctx.translate(handle)
    if nb == 0:
        return np.zeros(0, dtype=np.uint8)
    return ctx.tensor(handle).cpu().numpy()
