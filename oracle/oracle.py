"""TEST INFRASTRUCTURE ONLY — ctypes wrapper of oracle/checl_oracle.c.

Every function forwards to the C oracle (plain definition
§III-C over FORMAT.md); nothing here computes CRCs or layouts itself.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass
from typing import List, Sequence, Tuple

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "checl_oracle.c")
LIB = os.path.join(HERE, "libchecl_oracle.so")

SUCCESS, INVALID_VALUE, OUT_OF_HOST_MEMORY, BAD_IMAGE, CRC_MISMATCH = 0, -1, -5, -6, -7


def build(force: bool = False) -> str:
    """Compile the oracle (plain C99, -O2, single-threaded)."""
    stale = force or not os.path.exists(LIB) or any(
        os.path.getmtime(os.path.join(HERE, f)) > os.path.getmtime(LIB) for f in ("checl_oracle.c", "checl_oracle.h"))
    if stale:
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-std=c99", "-O2", "-Wall", "-Wextra", "-fPIC", "-shared", SRC, "-o", tmp])
        os.replace(tmp, LIB)
    return LIB


class _Buf(C.Structure):
    _fields_ = [("handle", C.c_uint64), ("size", C.c_uint64), ("flags", C.c_uint32),
                ("device", C.c_int32), ("data", C.c_void_p)]


class _Layout(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in ("n_buffers", "n_chunks", "crc_off", "payload_off", "payload_bytes", "image_bytes")]


class Report(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in ("n_buffers", "payload_bytes", "n_chunks", "n_bad_chunks",
                                          "first_bad_handle", "first_bad_chunk")]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n, _ in self._fields_}


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        _lib.oracle_crc32c.restype = C.c_uint32
        _lib.oracle_crc32c.argtypes = [C.c_void_p, C.c_size_t]
        _lib.oracle_crc32c_bitwise.restype = C.c_uint32
        _lib.oracle_crc32c_bitwise.argtypes = [C.c_void_p, C.c_size_t]
        _lib.oracle_layout_of.argtypes = [C.POINTER(_Buf), C.c_size_t, C.POINTER(_Layout)]
        _lib.oracle_checkpoint.argtypes = [C.POINTER(_Buf), C.c_size_t, C.c_int32, C.c_uint64, C.c_void_p, C.c_size_t]
        _lib.oracle_validate.argtypes = [C.c_void_p, C.c_size_t, C.POINTER(Report)]
        _lib.oracle_restore.argtypes = [C.c_void_p, C.c_size_t, C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p,
                                        C.c_void_p, C.c_size_t, C.POINTER(Report)]
    return _lib


def _u8(b) -> np.ndarray:
    if isinstance(b, (bytes, bytearray, memoryview)):
        return np.frombuffer(bytes(b), dtype=np.uint8)
    return np.ascontiguousarray(b).view(np.uint8).reshape(-1)


def crc32c(data) -> int:
    a = _u8(data)
    return int(lib().oracle_crc32c(a.ctypes.data if a.size else None, a.size))


def crc32c_bitwise(data) -> int:
    a = _u8(data)
    return int(lib().oracle_crc32c_bitwise(a.ctypes.data if a.size else None, a.size))


@dataclass
class Entry:
    """A live registry entry: (handle, bytes, flags)."""
    handle: int
    data: np.ndarray  # uint8
    flags: int = 0


def _bufs(entries: Sequence[Entry], device: int):
    arr = (_Buf * max(1, len(entries)))()
    keep = []
    for i, e in enumerate(entries):
        d = _u8(e.data)
        keep.append(d)
        arr[i] = _Buf(e.handle, d.size, e.flags, device, d.ctypes.data if d.size else None)
    return arr, keep


def layout(sizes_by_handle: Sequence[Tuple[int, int]]) -> dict:
    """Layout for [(handle, size), ...] without data (data pointers are dummies)."""
    dummy = np.zeros(1, dtype=np.uint8)
    arr = (_Buf * max(1, len(sizes_by_handle)))()
    for i, (h, s) in enumerate(sizes_by_handle):
        arr[i] = _Buf(h, s, 0, 0, dummy.ctypes.data)
    L = _Layout()
    st = lib().oracle_layout_of(arr, len(sizes_by_handle), C.byref(L))
    if st:
        raise ValueError(f"oracle_layout_of status {st}")
    return {n: int(getattr(L, n)) for n, _ in L._fields_}


def checkpoint(entries: Sequence[Entry], device: int = 0, epoch: int = 0) -> np.ndarray:
    arr, keep = _bufs(entries, device)
    L = _Layout()
    st = lib().oracle_layout_of(arr, len(entries), C.byref(L))
    if st:
        raise ValueError(f"oracle_layout_of status {st}")
    out = np.empty(L.image_bytes, dtype=np.uint8)
    st = lib().oracle_checkpoint(arr, len(entries), device, epoch, out.ctypes.data, out.size)
    if st:
        raise ValueError(f"oracle_checkpoint status {st}")
    return out


def validate(img) -> Tuple[int, dict]:
    a = _u8(img)
    rep = Report()
    st = lib().oracle_validate(a.ctypes.data if a.size else None, a.size, C.byref(rep))
    return int(st), rep.as_dict()


def restore(img) -> Tuple[int, dict, List[Entry]]:
    """Returns (status, report, [Entry(handle, bytes, flags)]) — entries empty unless SUCCESS."""
    a = _u8(img)
    st, rep = validate(a)
    if st:
        return st, rep, []
    n = rep["n_buffers"]
    hs = np.zeros(max(1, n), dtype=np.uint64)
    ss = np.zeros(max(1, n), dtype=np.uint64)
    fs = np.zeros(max(1, n), dtype=np.uint32)
    total = rep["payload_bytes"]  # upper bound of Σ sizes
    out = np.empty(max(1, total), dtype=np.uint8)
    r = Report()
    st = lib().oracle_restore(a.ctypes.data, a.size, out.ctypes.data, out.size, hs.ctypes.data, ss.ctypes.data,
                              fs.ctypes.data, n, C.byref(r))
    if st:
        return int(st), r.as_dict(), []
    ents, pos = [], 0
    for i in range(n):
        s = int(ss[i])
        ents.append(Entry(int(hs[i]), out[pos:pos + s].copy(), int(fs[i])))
        pos += s
    return 0, r.as_dict(), ents


def _sigs_incremental(L):
    if getattr(L, "_incr", False):
        return L
    L.oracle_checkpoint_incremental.argtypes = [C.POINTER(_Buf), C.c_size_t, C.c_int32, C.c_uint64, C.c_void_p,
                                                C.c_size_t, C.c_void_p, C.c_size_t, C.POINTER(C.c_uint64)]
    L.oracle_checkpoint_incremental_rule.argtypes = [C.POINTER(_Buf), C.c_size_t, C.c_int32, C.c_uint64, C.c_void_p,
                                                     C.c_size_t, C.c_void_p, C.c_size_t, C.c_uint32, C.c_void_p,
                                                     C.c_size_t, C.POINTER(C.c_uint64)]
    L.oracle_merge.argtypes = [C.c_void_p, C.c_size_t, C.c_void_p, C.c_size_t, C.c_void_p, C.c_size_t,
                               C.POINTER(C.c_uint64)]
    L._incr = True
    return L


RULE_CRC, RULE_BYTES = 0, 1  # FORMAT.md "Present set" (readings 21 and 25)


def checkpoint_incremental(entries: Sequence[Entry], base, device: int = 0, epoch: int = 0, rule: int = RULE_CRC,
                           base_full=None) -> np.ndarray:
    """Incremental image of the registry relative to `base` (FORMAT.md "Incremental
    images"); the full image when the layout differs from the base's. rule=RULE_BYTES
    needs base_full, the full image of the base's state (base itself when full)."""
    L = _sigs_incremental(lib())
    arr, keep = _bufs(entries, device)
    b = _u8(base)
    f = _u8(base_full) if base_full is not None else None
    fp, fn = (f.ctypes.data if f is not None and f.size else None), (f.size if f is not None else 0)
    need = C.c_uint64(0)
    st = L.oracle_checkpoint_incremental_rule(arr, len(entries), device, epoch, b.ctypes.data if b.size else None,
                                              b.size, fp, fn, rule, None, 0, C.byref(need))
    if st != INVALID_VALUE or need.value == 0:  # cap 0: reports the size it needs
        raise ValueError(f"oracle_checkpoint_incremental status {st}")
    out = np.empty(max(1, need.value), dtype=np.uint8)
    st = L.oracle_checkpoint_incremental_rule(arr, len(entries), device, epoch, b.ctypes.data if b.size else None,
                                              b.size, fp, fn, rule, out.ctypes.data, out.size, C.byref(need))
    if st:
        raise ValueError(f"oracle_checkpoint_incremental status {st}")
    return out[: need.value]


def merge(full, delta) -> Tuple[int, np.ndarray]:
    """(status, merge(F, D)) — the full image of D's epoch (FORMAT.md "Merge")."""
    L = _sigs_incremental(lib())
    f, d = _u8(full), _u8(delta)
    need = C.c_uint64(0)
    st = L.oracle_merge(f.ctypes.data, f.size, d.ctypes.data, d.size, None, 0, C.byref(need))
    if st != INVALID_VALUE:
        return int(st), np.zeros(0, np.uint8)
    out = np.empty(max(1, need.value), dtype=np.uint8)
    st = L.oracle_merge(f.ctypes.data, f.size, d.ctypes.data, d.size, out.ctypes.data, out.size, C.byref(need))
    return int(st), out[: need.value]


def restore_chain(chain) -> Tuple[int, dict, List[Entry]]:
    """Restores [F, D1, ..., Dn] as restore(merge(...merge(F, D1)..., Dn))."""
    cur = _u8(chain[0])
    for d in chain[1:]:
        st, cur = merge(cur, d)
        if st:
            return st, {}, []
    return restore(cur)
