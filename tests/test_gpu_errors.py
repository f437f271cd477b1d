"""-m gpu: error paths of the C ABI on a real device — allocator failure leaves every
handle bound where it was (OUT_OF_DEVICE_MEMORY, all-or-nothing restore, L16
restart step 2 cannot re-create the objects), a concurrent checkpoint on one
context is refused (BUSY), and the cudaMalloc allocator path restores bit-exact."""
import ctypes as C
import threading
import time

import numpy as np
import pytest

from oracle import oracle as O
from tests.gpu_util import bound_bytes, make_set, oracle_entries, release_all

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

DEV = 0


def test_allocator_failure_rebinds_nothing():
    state = {"fail": False, "allocs": 0}

    @C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)
    def _alloc(nbytes, device, stream, user):
        state["allocs"] += 1
        if state["fail"]:
            return None
        return torch.cuda.caching_allocator_alloc(int(nbytes), device, int(stream or 0))

    @C.CFUNCTYPE(None, C.c_void_p, C.c_int, C.c_void_p, C.c_void_p)
    def _free(ptr, device, stream, user):
        torch.cuda.caching_allocator_delete(int(ptr))

    ctx = checl.Context(allocator=checl.Allocator(_alloc, _free, None))
    ds = make_set(ctx, [300007, 17, 65536], seed=41)
    img = ctx.checkpoint(DEV, epoch=1)
    before = [ctx.translate(h) for h in ds.handles]
    state["fail"] = True
    with pytest.raises(checl.CheclError) as ei:
        ctx.restore(img, DEV)
    assert ei.value.status == checl.ERR_OUT_OF_DEVICE_MEMORY
    assert [ctx.translate(h) for h in ds.handles] == before  # nothing rebound
    state["fail"] = False
    rep = ctx.restore(img, DEV)  # the context is still usable
    assert rep.n_bad_chunks == 0
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)
    ctx.close()


def test_concurrent_checkpoint_is_busy():
    ctx = checl.Context()
    big = torch.empty(2 << 30, dtype=torch.uint8, device=DEV)
    checl.debug_fill(big, 3, 0)
    torch.cuda.synchronize()
    ctx.register(big)
    img = ctx.checkpoint(DEV, epoch=0)  # pins the host image once
    errs = []

    def worker():
        try:
            for e in range(3):
                ctx.checkpoint(DEV, epoch=e, into=img)
        except Exception as ex:  # noqa: BLE001
            errs.append(ex)

    t = threading.Thread(target=worker)
    t.start()
    time.sleep(0.01)
    busy = 0
    deadline = time.time() + 5
    while t.is_alive() and time.time() < deadline:
        try:
            ctx.checkpoint(DEV, epoch=99, into=img)
        except checl.CheclError as e:
            assert e.status == checl.ERR_BUSY
            busy += 1
            time.sleep(0.002)
    t.join()
    assert not errs and busy > 0
    img.free()
    ctx.close()


def test_cudamalloc_allocator_round_trip():
    ctx = checl.Context(allocator="cuda")
    ds = make_set(ctx, [70001, 0, 1 << 20], seed=42, offsets=[3, 0, 0])
    img = ctx.checkpoint(DEV, epoch=2)
    assert np.array_equal(img.view(), O.checkpoint(oracle_entries(ds), device=DEV, epoch=2))
    ctx.restore(img, DEV)
    ctx.restore(img, DEV)  # the first restore's allocation is released / reused
    ctx.trim()             # spares and pooled pinned buffers released
    ctx.restore(img, DEV)
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)
    release_all(ctx, ds)
    ctx.close()
