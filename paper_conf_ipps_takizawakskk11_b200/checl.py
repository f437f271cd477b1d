"""Python binding of libchecl (include/checl.h) — argument marshalling only.

Every step of the snapshot path (database walk, pack + CRC32C, drain, fill,
verify + scatter, rebind) runs in libchecl.so; this module converts tensors to
pointers, images to numpy views, and status codes to exceptions. PyTorch is used
for device memory (the caching allocator backs re-created buffers), streams and
process groups. There is no fallback: if libchecl.so is missing, importing this
module raises.

Paper anchors: CheCL handles and translation L15 §III-B; the object
database L19 §III-C; checkpoint/restart steps L16 §III-C; migration L40 §IV-C.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass
from typing import Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("CHECL_LIB", os.path.join(_HERE, "libchecl.so"))  # override: experiments only

SUCCESS = 0
ERR_INVALID_VALUE = -1
ERR_INVALID_HANDLE = -2
ERR_INVALID_DEVICE = -3
ERR_OUT_OF_DEVICE_MEMORY = -4
ERR_OUT_OF_HOST_MEMORY = -5
ERR_BAD_IMAGE = -6
ERR_CRC_MISMATCH = -7
ERR_CUDA = -8
ERR_PEER_ACCESS = -9
ERR_BUSY = -10

IMAGE_HOST, IMAGE_DEVICE = 0, 1
IO_DIRECT, IO_SYNC = 1, 2
FILL_RANDOM, FILL_FLOAT, FILL_ZEROS = 0, 1, 2
DIRTY_CRC, DIRTY_BYTES = 0, 1  # incremental checkpoint dirty rules (checl.h, FORMAT.md "Present set")

EXPORTS = (
    "checl_create", "checl_destroy", "checl_set_staging", "checl_register_buffer", "checl_release",
    "checl_translate", "checl_count", "checl_checkpoint", "checl_checkpoint_into", "checl_checkpoint_device",
    "checl_image_view", "checl_image_info", "checl_image_wrap", "checl_image_to_host", "checl_image_free",
    "checl_restore", "checl_migrate", "checl_last_timing", "checl_status_string", "checl_last_cuda_error",
    "checl_version", "checl_debug_fill", "checl_debug_compare", "checl_debug_corrupt",
    "checl_checkpoint_incremental", "checl_checkpoint_incremental_ex", "checl_restore_chain", "checl_image_merge",
    "checl_request_checkpoint", "checl_checkpoint_pending", "checl_install_signal", "checl_sync_point",
    "checl_image_write", "checl_image_read", "checl_trim", "checl_stats_get", "checl_stats_reset",
)


class Allocator(C.Structure):
    _fields_ = [("alloc", C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)),
                ("free", C.CFUNCTYPE(None, C.c_void_p, C.c_int, C.c_void_p, C.c_void_p)),
                ("user", C.c_void_p)]


class _Report(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in ("n_buffers", "payload_bytes", "n_chunks", "n_bad_chunks",
                                          "first_bad_handle", "first_bad_chunk")]


class _Timing(C.Structure):
    _fields_ = [("sync_ms", C.c_double), ("plan_ms", C.c_double), ("alloc_ms", C.c_double),
                ("kernel_ms", C.c_double), ("copy_ms", C.c_double), ("commit_ms", C.c_double),
                ("total_ms", C.c_double), ("n_stages", C.c_uint64), ("n_kernels", C.c_uint64)]


class _Stats(C.Structure):
    _fields_ = [("n_calls", C.c_uint64), ("total_ms", C.c_double), ("kernel_ms", C.c_double),
                ("copy_ms", C.c_double), ("n_kernels", C.c_uint64)]


STATS_CHECKPOINT, STATS_RESTORE, STATS_INCREMENTAL, STATS_CHAIN = 0, 1, 2, 3


def _load() -> C.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is not built: run `python -m paper_conf_ipps_takizawakskk11_b200.build` "
                          "(there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    P, V, U64, I32, U32, SZ = C.c_void_p, C.c_void_p, C.c_uint64, C.c_int32, C.c_uint32, C.c_size_t
    PP = C.POINTER(C.c_void_p)
    sig = {
        "checl_create": [C.POINTER(Allocator), PP],
        "checl_destroy": [P],
        "checl_set_staging": [P, SZ, U32],
        "checl_register_buffer": [P, C.c_int, V, SZ, U32, C.POINTER(U64)],
        "checl_release": [P, U64],
        "checl_translate": [P, U64, PP, C.POINTER(SZ), C.POINTER(C.c_int)],
        "checl_count": [P, C.c_int, C.POINTER(U64), C.POINTER(U64)],
        "checl_checkpoint": [P, C.c_int, V, U64, PP],
        "checl_checkpoint_into": [P, C.c_int, V, U64, P],
        "checl_checkpoint_device": [P, C.c_int, V, U64, PP],
        "checl_image_view": [P, PP, C.POINTER(SZ)],
        "checl_image_info": [P, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(U64), PP],
        "checl_image_wrap": [V, SZ, PP],
        "checl_image_to_host": [P, PP],
        "checl_image_free": [P],
        "checl_restore": [P, P, C.c_int, V, C.POINTER(_Report)],
        "checl_migrate": [P, C.c_int, C.c_int, V, C.POINTER(_Report)],
        "checl_last_timing": [P, C.POINTER(_Timing)],
        "checl_stats_get": [P, C.c_int, C.POINTER(_Stats)],
        "checl_stats_reset": [P],
        "checl_debug_fill": [C.c_int, V, SZ, U64, U64, C.c_int, V],
        "checl_debug_compare": [C.c_int, V, V, SZ, C.POINTER(U64)],
        "checl_debug_corrupt": [P, U64, C.c_uint8],
        "checl_checkpoint_incremental": [P, C.c_int, V, U64, P, PP],
        "checl_checkpoint_incremental_ex": [P, C.c_int, V, U64, P, U32, PP],
        "checl_restore_chain": [P, C.POINTER(C.c_void_p), U32, C.c_int, V, C.POINTER(_Report)],
        "checl_image_merge": [P, P, PP],
        "checl_request_checkpoint": [P],
        "checl_checkpoint_pending": [P, C.POINTER(C.c_int)],
        "checl_install_signal": [P, C.c_int],
        "checl_sync_point": [P, C.c_int, V, U64, P, PP],
        "checl_image_write": [P, C.c_char_p, U32],
        "checl_image_read": [C.c_char_p, U32, PP],
        "checl_trim": [P],
    }
    for name, args in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = I32
    lib.checl_status_string.argtypes = [I32]
    lib.checl_status_string.restype = C.c_char_p
    lib.checl_last_cuda_error.argtypes = []
    lib.checl_last_cuda_error.restype = C.c_char_p
    lib.checl_version.argtypes = []
    lib.checl_version.restype = U32
    return lib


lib = _load()


class CheclError(RuntimeError):
    def __init__(self, status: int, what: str = "", report: Optional["Report"] = None):
        name = lib.checl_status_string(status).decode()
        extra = ""
        if status == ERR_CUDA:
            extra = f" ({lib.checl_last_cuda_error().decode()})"
        super().__init__(f"{what}: {name}{extra}")
        self.status = status
        self.report = report


def _check(st: int, what: str, report=None):
    if st != SUCCESS:
        raise CheclError(st, what, report)


@dataclass
class Report:
    n_buffers: int
    payload_bytes: int
    n_chunks: int
    n_bad_chunks: int
    first_bad_handle: int
    first_bad_chunk: int

    @classmethod
    def _from(cls, r: _Report) -> "Report":
        return cls(*(int(getattr(r, n)) for n, _ in _Report._fields_))


def _stream_ptr(stream) -> Optional[int]:
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream or None
    return stream.cuda_stream or None  # torch.cuda.Stream


class Image:
    """A checkpoint image (FORMAT.md). Host images expose their bytes as a numpy
    view; device images keep payload + CRC table in HBM (view() = the metadata
    mirror [0, payload_off))."""

    def __init__(self, ptr: int, keepalive=None):
        self._p = C.c_void_p(ptr)
        self._keep = keepalive

    @property
    def handle(self) -> C.c_void_p:
        if not self._p:
            raise ValueError("image freed")
        return self._p

    @classmethod
    def wrap(cls, data) -> "Image":
        """Borrow caller bytes (numpy uint8 / bytes) as an image (no copy)."""
        arr = np.ascontiguousarray(np.frombuffer(data, dtype=np.uint8) if isinstance(data, (bytes, bytearray)) else data)
        arr = arr.view(np.uint8).reshape(-1)
        out = C.c_void_p()
        _check(lib.checl_image_wrap(arr.ctypes.data if arr.size else None, arr.size, C.byref(out)), "checl_image_wrap")
        return cls(out.value, keepalive=arr)

    def info(self) -> dict:
        loc, dev, nb, pay = C.c_int(), C.c_int(), C.c_uint64(), C.c_void_p()
        _check(lib.checl_image_info(self.handle, C.byref(loc), C.byref(dev), C.byref(nb), C.byref(pay)), "checl_image_info")
        return {"location": loc.value, "device": dev.value, "image_bytes": nb.value, "device_payload": pay.value}

    def view(self) -> np.ndarray:
        b, n = C.c_void_p(), C.c_size_t()
        _check(lib.checl_image_view(self.handle, C.byref(b), C.byref(n)), "checl_image_view")
        if n.value == 0:
            return np.zeros(0, dtype=np.uint8)
        # the array keeps this Image alive (a view of a temporary, e.g. a.merge(d).view(),
        # must not outlive the image's memory); free() still ends it
        buf = (C.c_uint8 * n.value).from_address(b.value)
        buf._image = self
        arr = np.frombuffer(buf, dtype=np.uint8)
        arr.flags.writeable = False
        return arr

    def merge(self, delta: "Image") -> "Image":
        """FORMAT.md "Merge": the full image of `delta`'s epoch (self = the full base)."""
        out = C.c_void_p()
        _check(lib.checl_image_merge(self.handle, delta.handle, C.byref(out)), "checl_image_merge")
        return Image(out.value)

    def header(self) -> dict:
        """Header fields (FORMAT.md) read from the image bytes."""
        v = self.view()
        u32 = lambda o: int(v[o:o + 4].view("<u4")[0])  # noqa: E731
        u64 = lambda o: int(v[o:o + 8].view("<u8")[0])  # noqa: E731
        h = {"n_buffers": u64(24), "n_chunks": u64(32), "crc_off": u64(48), "payload_off": u64(56),
             "payload_bytes": u64(64), "image_bytes": u64(72), "device": u32(80), "flags": u32(84), "epoch": u64(88)}
        if h["flags"] == 1:
            h.update(base_epoch=u64(96), base_table_crc=u32(104), dirty_rule=u32(108), n_present=u64(112))
        return h

    def write(self, path: str, direct: bool = True, sync: bool = False):
        """Writing phase (L16 step 3 analogue): the image bytes to a file."""
        _check(lib.checl_image_write(self.handle, os.fsencode(path), (IO_DIRECT if direct else 0) | (IO_SYNC if sync else 0)),
               "checl_image_write")

    @classmethod
    def read(cls, path: str, direct: bool = True) -> "Image":
        """An image file read back into a (pinned) host image; metadata validated."""
        out = C.c_void_p()
        _check(lib.checl_image_read(os.fsencode(path), IO_DIRECT if direct else 0, C.byref(out)), "checl_image_read")
        return cls(out.value)

    def to_host(self) -> "Image":
        out = C.c_void_p()
        _check(lib.checl_image_to_host(self.handle, C.byref(out)), "checl_image_to_host")
        return Image(out.value)

    def corrupt(self, image_offset: int, mask: int):
        """Fault injection (tests): XOR mask into one byte of the image."""
        _check(lib.checl_debug_corrupt(self.handle, image_offset, mask), "checl_debug_corrupt")

    def free(self):
        if self._p:
            lib.checl_image_free(self._p)
            self._p = C.c_void_p()
            self._keep = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def _torch_allocator():
    import torch

    @C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)
    def _alloc(nbytes, device, stream, user):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), device, int(stream or 0))
        except Exception:
            return None

    @C.CFUNCTYPE(None, C.c_void_p, C.c_int, C.c_void_p, C.c_void_p)
    def _free(ptr, device, stream, user):
        try:
            torch.cuda.caching_allocator_delete(int(ptr))
        except Exception:
            pass

    return Allocator(_alloc, _free, None)


class Context:
    """The CheCL object database + handle table of one process (L15, L19)."""

    def __init__(self, allocator="torch", slot_bytes: Optional[int] = None, n_slots: int = 2):
        """allocator: "torch" (the caching allocator), "cuda" (cudaMalloc / cudaFree),
        or an `Allocator` struct of C callbacks (kept alive by the context)."""
        if isinstance(allocator, Allocator):
            self._alloc = allocator
        else:
            self._alloc = _torch_allocator() if allocator == "torch" else None
        out = C.c_void_p()
        _check(lib.checl_create(C.byref(self._alloc) if self._alloc is not None else None, C.byref(out)), "checl_create")
        self._p = out
        if slot_bytes is not None:
            self.set_staging(slot_bytes, n_slots)

    # -- lifecycle
    def close(self):
        if getattr(self, "_p", None):
            lib.checl_destroy(self._p)
            self._p = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_staging(self, slot_bytes: int, n_slots: int = 2):
        _check(lib.checl_set_staging(self._p, slot_bytes, n_slots), "checl_set_staging")

    # -- object database / handle table
    def register_ptr(self, device: int, ptr: int, nbytes: int, flags: int = 0) -> int:
        h = C.c_uint64()
        _check(lib.checl_register_buffer(self._p, device, ptr or None, nbytes, flags, C.byref(h)), "checl_register_buffer")
        return h.value

    def register(self, tensor, flags: int = 0) -> int:
        """Registers a CUDA tensor's bytes (any view; must be contiguous)."""
        if not tensor.is_cuda:
            raise ValueError("register() takes CUDA tensors")
        if not tensor.is_contiguous():
            raise ValueError("register() takes contiguous tensors")
        nbytes = tensor.numel() * tensor.element_size()
        return self.register_ptr(tensor.device.index, tensor.data_ptr() if nbytes else 0, nbytes, flags)

    def release(self, handle: int):
        _check(lib.checl_release(self._p, handle), "checl_release")

    def translate(self, handle: int) -> Tuple[int, int, int]:
        ptr, nb, dev = C.c_void_p(), C.c_size_t(), C.c_int()
        _check(lib.checl_translate(self._p, handle, C.byref(ptr), C.byref(nb), C.byref(dev)), "checl_translate")
        return (ptr.value or 0, nb.value, dev.value)

    def tensor(self, handle: int, dtype=None, shape=None):
        """A torch view of the buffer a handle is currently bound to (uint8 by default)."""
        import torch
        ptr, nb, dev = self.translate(handle)
        dtype = dtype or torch.uint8
        esize = torch.empty(0, dtype=dtype).element_size()
        if shape is None:
            shape = (nb // esize,)
        typestr = {torch.uint8: "|u1", torch.float32: "<f4", torch.float64: "<f8", torch.int32: "<i4",
                   torch.int64: "<i8", torch.int8: "|i1", torch.float16: "<f2"}[dtype]

        class _Iface:
            __cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (ptr, False),
                                        "version": 2, "strides": None}
        with torch.cuda.device(dev):
            return torch.as_tensor(_Iface(), device=f"cuda:{dev}")

    def count(self, device: int) -> Tuple[int, int]:
        n, t = C.c_uint64(), C.c_uint64()
        _check(lib.checl_count(self._p, device, C.byref(n), C.byref(t)), "checl_count")
        return n.value, t.value

    # -- checkpoint / restore / migrate
    def checkpoint(self, device: int, stream=None, epoch: int = 0, into: Optional[Image] = None) -> Image:
        """Immediate-mode checkpoint (L16 steps 1-2) into a pinned host image."""
        if into is not None:
            _check(lib.checl_checkpoint_into(self._p, device, _stream_ptr(stream), epoch, into.handle), "checl_checkpoint_into")
            return into
        out = C.c_void_p()
        _check(lib.checl_checkpoint(self._p, device, _stream_ptr(stream), epoch, C.byref(out)), "checl_checkpoint")
        return Image(out.value)

    def checkpoint_device(self, device: int, stream=None, epoch: int = 0) -> Image:
        """Checkpoint into an image resident in the device's HBM."""
        out = C.c_void_p()
        _check(lib.checl_checkpoint_device(self._p, device, _stream_ptr(stream), epoch, C.byref(out)),
               "checl_checkpoint_device")
        return Image(out.value)

    def checkpoint_incremental(self, device: int, base: Image, stream=None, epoch: int = 0,
                               rule: int = DIRTY_BYTES) -> Image:
        """Incremental checkpoint (L45 future work; FORMAT.md "Incremental images"):
        only the updated chunks are drained — rule DIRTY_BYTES (default, exact): the
        chunks whose bytes differ from `base`'s state; DIRTY_CRC (fast option): the
        chunks whose CRC32C differs from `base`'s table."""
        out = C.c_void_p()
        _check(lib.checl_checkpoint_incremental_ex(self._p, device, _stream_ptr(stream), epoch, base.handle, rule,
                                                   C.byref(out)), "checl_checkpoint_incremental_ex")
        return Image(out.value)

    def restore_chain(self, chain, device: int, stream=None) -> Report:
        """Restores [full, delta1, ..., deltaN] (all or nothing)."""
        arr = (C.c_void_p * len(chain))(*[im.handle.value for im in chain])
        r = _Report()
        st = lib.checl_restore_chain(self._p, arr, len(chain), device, _stream_ptr(stream), C.byref(r))
        rep = Report._from(r)
        _check(st, "checl_restore_chain", rep)
        return rep

    def restore(self, image: Image, device: int, stream=None, report: bool = True) -> Optional[Report]:
        """Restart steps 2-3 (L16): verify every chunk, then rebind every handle.
        report=False passes no report (the call's status alone; a hot loop skips
        building the Report)."""
        if not report:
            _check(lib.checl_restore(self._p, image.handle, device, _stream_ptr(stream), None), "checl_restore")
            return None
        r = _Report()
        st = lib.checl_restore(self._p, image.handle, device, _stream_ptr(stream), C.byref(r))
        rep = Report._from(r)
        _check(st, "checl_restore", rep)
        return rep

    def migrate(self, src_device: int, dst_device: int, stream=None) -> Report:
        r = _Report()
        st = lib.checl_migrate(self._p, src_device, dst_device, _stream_ptr(stream), C.byref(r))
        rep = Report._from(r)
        _check(st, "checl_migrate", rep)
        return rep

    # -- delayed checkpointing mode (L16 §III-C)
    def request_checkpoint(self):
        _check(lib.checl_request_checkpoint(self._p), "checl_request_checkpoint")

    def checkpoint_pending(self) -> bool:
        v = C.c_int()
        _check(lib.checl_checkpoint_pending(self._p, C.byref(v)), "checl_checkpoint_pending")
        return bool(v.value)

    def install_signal(self, signo: int):
        """A handler for `signo` (e.g. signal.SIGUSR1) that requests a checkpoint."""
        _check(lib.checl_install_signal(self._p, signo), "checl_install_signal")

    def sync_point(self, device: int, stream=None, epoch: int = 0, into: Optional[Image] = None) -> Optional[Image]:
        """clFinish analogue: synchronises `stream`; checkpoints iff one was requested."""
        out = C.c_void_p()
        _check(lib.checl_sync_point(self._p, device, _stream_ptr(stream), epoch, into.handle if into else None,
                                    C.byref(out)), "checl_sync_point")
        if not out.value:
            return None
        return into if into is not None else Image(out.value)

    def trim(self):
        """Release the spare allocations and pooled pinned buffers kept for reuse."""
        _check(lib.checl_trim(self._p), "checl_trim")

    def last_timing(self, raw: bool = False):
        """Phase times of the last checkpoint / restore (checl_timing); raw=True returns
        the ctypes struct (cheap inside a timed loop; convert with timing_dict)."""
        t = _Timing()
        _check(lib.checl_last_timing(self._p, C.byref(t)), "checl_last_timing")
        return t if raw else timing_dict(t)

    def stats(self, kind: int) -> dict:
        """Cumulative timing of one kind of call (STATS_*) since creation / reset_stats."""
        t = _Stats()
        _check(lib.checl_stats_get(self._p, kind, C.byref(t)), "checl_stats_get")
        return _stats_dict(t)

    def reset_stats(self):
        _check(lib.checl_stats_reset(self._p), "checl_stats_reset")


def _stats_dict(t) -> dict:
    return {n: (float(getattr(t, n)) if ty is C.c_double else int(getattr(t, n))) for n, ty in _Stats._fields_}


def timing_dict(t) -> dict:
    return {n: (float(getattr(t, n)) if ty is C.c_double else int(getattr(t, n))) for n, ty in _Timing._fields_}


# -- test / bench tooling -----------------------------------------------------------

def debug_fill(tensor, seed: int, stream_id: int, kind: int = FILL_RANDOM, stream=None):
    """Fill a CUDA tensor's bytes with the synth/ generator, on the device."""
    nbytes = tensor.numel() * tensor.element_size()
    _check(lib.checl_debug_fill(tensor.device.index, tensor.data_ptr() if nbytes else None, nbytes, seed, stream_id, kind,
                                _stream_ptr(stream)), "checl_debug_fill")


def debug_fill_ptr(device: int, ptr: int, nbytes: int, seed: int, stream_id: int, kind: int = FILL_RANDOM, stream=None):
    _check(lib.checl_debug_fill(device, ptr or None, nbytes, seed, stream_id, kind, _stream_ptr(stream)), "checl_debug_fill")


def debug_compare(device: int, a_ptr: int, b_ptr: int, nbytes: int) -> int:
    n = C.c_uint64()
    _check(lib.checl_debug_compare(device, a_ptr or None, b_ptr or None, nbytes, C.byref(n)), "checl_debug_compare")
    return n.value


def version() -> int:
    return int(lib.checl_version())
