"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

Holds NONE of the method's arithmetic (no CRC, no layout, no packing): only
buffer-size recipes shaped like the paper's workloads (DESIGN.md
§4) and a counter-based byte generator. The CUDA library implements the same
generator as a device fill kernel (test tooling, `checl_debug_fill`), so device
buffers never need a host copy to be filled; tests compare the two generators.

Generator (splitmix64 finaliser over a per-buffer counter):
    state_i = key + (i + 1) * GOLDEN            (mod 2^64)
    word_i  = mix64(state_i)
    key     = mix64(seed * GOLDEN ^ (stream + 1) * KEYMUL)
    bytes   = little-endian words, truncated to the buffer size
kinds: "random" (the words as is), "float" (each 32-bit half becomes a float32
in [0,1): (half >> 8) * 2^-24), "zeros".
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List

import numpy as np

GOLDEN = 0x9E3779B97F4A7C15
KEYMUL = 0xD1B54A32D192ED03
M64 = (1 << 64) - 1
KINDS = {"random": 0, "float": 1, "zeros": 2}


def mix64(z: int) -> int:
    z &= M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def stream_key(seed: int, stream: int) -> int:
    return mix64(((seed * GOLDEN) & M64) ^ (((stream + 1) * KEYMUL) & M64))


def u64_at(seed: int, stream: int, i: int) -> int:
    """Scalar draw: word i of (seed, stream)."""
    return mix64((stream_key(seed, stream) + (i + 1) * GOLDEN) & M64)


def _mix64_np(z: np.ndarray) -> np.ndarray:
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def fill_slice(offset: int, length: int, seed: int, stream: int, kind: str = "random") -> np.ndarray:
    """Bytes [offset, offset + length) of a buffer filled by fill_bytes (counter-based:
    no need to generate the prefix)."""
    w0 = offset // 8
    head = offset - 8 * w0
    b = fill_bytes(head + length, seed, stream, kind, word0=w0)
    return b[head:head + length]


def fill_bytes(size: int, seed: int, stream: int, kind: str = "random", out: np.ndarray | None = None,
               word0: int = 0) -> np.ndarray:
    """Host copy of the bytes the device fill kernel writes (uint8[size]); with
    word0 > 0, the bytes starting at word word0 of the buffer."""
    if out is None:
        out = np.empty(size, dtype=np.uint8)
    if size == 0:
        return out
    if kind == "zeros":
        out[:] = 0
        return out
    nwords = (size + 7) // 8
    key = np.uint64(stream_key(seed, stream))
    step = 1 << 22  # bounded temporaries
    for w0 in range(0, nwords, step):
        w1 = min(nwords, w0 + step)
        with np.errstate(over="ignore"):
            st = key + (np.arange(word0 + w0 + 1, word0 + w1 + 1, dtype=np.uint64) * np.uint64(GOLDEN))
            words = _mix64_np(st)
        if kind == "float":
            lo = (words & np.uint64(0xFFFFFFFF)).astype(np.uint32) >> np.uint32(8)
            hi = (words >> np.uint64(32)).astype(np.uint32) >> np.uint32(8)
            f = np.empty((w1 - w0, 2), dtype=np.float32)
            f[:, 0] = lo.astype(np.float32) * np.float32(2.0 ** -24)
            f[:, 1] = hi.astype(np.float32) * np.float32(2.0 ** -24)
            b = f.view(np.uint8).reshape(-1)
        else:
            b = words.view(np.uint8)
        lo_b = w0 * 8
        hi_b = min(size, w1 * 8)
        out[lo_b:hi_b] = b[: hi_b - lo_b]
    return out


@dataclass
class BufferSpec:
    name: str
    size: int
    stream: int
    flags: int = 0


@dataclass
class Workload:
    name: str
    seed: int
    buffers: List[BufferSpec] = field(default_factory=list)

    @property
    def total_bytes(self) -> int:
        return sum(b.size for b in self.buffers)


def c1_vectoradd() -> Workload:
    """configs[0]: vectorAdd, 3 float32 buffers x 1 MiB (A, B, C = A + B)."""
    n = 262144 * 4
    return Workload("C1-vectorAdd", 1, [BufferSpec(nm, n, i) for i, nm in enumerate("ABC")])


def c2_sdk_mix() -> Workload:
    """configs[1]: SDK-sample mix (matrixMul, nbody, FDTD3d shapes), 463,040,532 B, 10 buffers."""
    f = 4
    sizes = [
        ("matrixMul.A", 800 * 480 * f), ("matrixMul.B", 480 * 1280 * f), ("matrixMul.C", 800 * 1280 * f),
        ("nbody.pos0", 30720 * 16), ("nbody.pos1", 30720 * 16), ("nbody.vel0", 30720 * 16), ("nbody.vel1", 30720 * 16),
        ("FDTD3d.in", 384 ** 3 * f), ("FDTD3d.out", 384 ** 3 * f), ("FDTD3d.coeff", 5 * f),
    ]
    return Workload("C2-SDK-mix", 2, [BufferSpec(nm, s, i) for i, (nm, s) in enumerate(sizes)])


def c3_handle_stress(n: int = 10000) -> Workload:
    """configs[2]: n odd-sized buffers, size_i = 4097 + 2 * (r_i mod 522240), r_i = draw(3, i)."""
    bufs = [BufferSpec(f"buf{i}", 4097 + 2 * (u64_at(3, 0, i) % 522240), i) for i in range(n)]
    return Workload("C3-handle-stress", 3, bufs)


def c4_md_rank(rank: int = 0, scale: float = 1.0) -> Workload:
    """configs[3]: SHOC-MD-shaped per-rank set; N = 126,322,567 atoms -> 68,719,476,448 B at scale 1."""
    natoms = int(126322567 * scale)
    return Workload(f"C4-MD-rank{rank}", 1000 + rank, [
        BufferSpec("md.pos", natoms * 16, 0), BufferSpec("md.force", natoms * 16, 1),
        BufferSpec("md.neigh", natoms * 4 * 128, 2)])


def c5_migration(large: bool = False) -> Workload:
    """configs[4]: migration set = the C2 set, or 16 x 1 GiB buffers."""
    if large:
        return Workload("C5-16GiB", 5, [BufferSpec(f"slab{i}", 1 << 30, i) for i in range(16)])
    w = c2_sdk_mix()
    w.name = "C5-SDK-mix"
    return w


CONFIGS = {"C1": c1_vectoradd, "C2": c2_sdk_mix, "C3": c3_handle_stress, "C4": c4_md_rank, "C5": c5_migration}
