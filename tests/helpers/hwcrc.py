"""Independent CRC32C implementations for pinning (test-only).

* `hw_crc32c`: the x86 SSE4.2 crc32 instruction (compiled on first use).
* `poly_crc32c`: the CRC as GF(2) polynomial remainder, with Python integers —
  a different mathematical formulation from the shift-register oracle:
      R(x) = (M(x) * x^32 + I(x) * x^(8n)) mod G(x),   I = all-ones (init),
  message bits taken LSB-first per byte, result complemented and bit-reflected.
"""
import ctypes as C
import os
import platform
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
_lib = None


def available() -> bool:
    return platform.machine() in ("x86_64", "AMD64")


def _load():
    global _lib
    if _lib is None:
        so = os.path.join(HERE, "libcrc32c_hw.so")
        src = os.path.join(HERE, "crc32c_hw.c")
        if not os.path.exists(so) or os.path.getmtime(src) > os.path.getmtime(so):
            tmp = so + f".tmp{os.getpid()}"
            subprocess.check_call(["gcc", "-O2", "-msse4.2", "-fPIC", "-shared", src, "-o", tmp])
            os.replace(tmp, so)
        _lib = C.CDLL(so)
        _lib.hw_crc32c.restype = C.c_uint32
        _lib.hw_crc32c.argtypes = [C.c_void_p, C.c_size_t]
        _lib.hw_crc32c_many.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p]
    return _lib


def hw_crc32c(data) -> int:
    a = np.frombuffer(bytes(data), dtype=np.uint8) if isinstance(data, (bytes, bytearray)) else np.ascontiguousarray(data).view(np.uint8).reshape(-1)
    return int(_load().hw_crc32c(a.ctypes.data if a.size else None, a.size))


def hw_crc32c_many(base: np.ndarray, offs, lens) -> np.ndarray:
    base = np.ascontiguousarray(base).view(np.uint8).reshape(-1)
    o = np.ascontiguousarray(offs, dtype=np.uint64)
    l = np.ascontiguousarray(lens, dtype=np.uint64)
    out = np.zeros(max(1, o.size), dtype=np.uint32)
    _load().hw_crc32c_many(base.ctypes.data, o.ctypes.data, l.ctypes.data, o.size, out.ctypes.data)
    return out[: o.size]


G = (1 << 32) | 0x1EDC6F41  # Castagnoli generator, normal (non-reflected) form


def _polymod(a: int, g: int = G) -> int:
    dg = g.bit_length() - 1
    while a.bit_length() - 1 >= dg:
        a ^= g << (a.bit_length() - 1 - dg)
    return a


def poly_crc32c(data: bytes) -> int:
    n = len(data)
    m = 0
    for byte in data:  # transmission order: LSB of each byte first
        for k in range(8):
            m = (m << 1) | ((byte >> k) & 1)
    r = _polymod((m << 32) ^ (0xFFFFFFFF << (8 * n)))
    r ^= 0xFFFFFFFF
    # coefficient of x^(31-j) becomes bit j of the reflected 32-bit value
    return int(f"{r:032b}"[::-1], 2)
