"""-m gpu: memory the library takes and gives back, and ordering against the caller's
stream.

* Migration is a move (§IV-C: a job "may better stop using GPUs and give
  them to other jobs"; reading 15): the source's migration image is freed
  as soon as K2 has read it, so after migrations plus checl_trim the device holds only
  the re-created buffers.
* Per-object release after restore (OpenCL objects are deleted one by one, L19-L20
  §III-C): restore re-creates the buffers in segments (reading 18), and a
  segment whose handles are all released goes back to the allocator.
* Restore into memory from the PyTorch caching allocator waits for the work the
  caller queued on its stream before that memory was handed out.
* A handle released on another thread while a checkpoint runs: the checkpoint still
  writes the bytes it planned (the release is deferred to the end of the call).
"""
import gc
import threading
import time

import numpy as np
import pytest

import synth
from oracle import oracle as O

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402
from tests.gpu_util import bound_bytes, make_set, oracle_entries  # noqa: E402

MiB = 1 << 20


def _held() -> int:
    """Bytes the caching allocator has handed out (the library's re-created buffers and
    migration images come from it): independent of how it caches segments. (Contexts
    of earlier tests left to the garbage collector are collected first: one collected
    mid-test would free its buffers inside the measured window.)"""
    gc.collect()
    torch.cuda.synchronize()
    return torch.cuda.memory_allocated(0)


def _used() -> int:
    """Device memory in use (cudaMemGetInfo) after the allocator returned its cache."""
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    free, total = torch.cuda.mem_get_info(0)
    return total - free


def test_migrate_frees_the_source_image():
    sizes = [64 * MiB + 5, 96 * MiB, 1 * MiB + 3, 64 * MiB]
    S = sum(sizes)
    with checl.Context() as ctx:
        ds = make_set(ctx, sizes, seed=31)
        probe = ctx.checkpoint_device(0, epoch=0)  # device state (tables, scratch) set up once
        probe.free()
        ctx.trim()
        before, used0 = _held(), _used()
        for _ in range(2):
            rep = ctx.migrate(0, 0)
            assert rep.n_bad_chunks == 0
        ctx.trim()
        after = _held()
        # the re-created buffers (S bytes, in 2 MiB-rounded blocks) are live; neither a
        # migration image nor the first migration's buffers are held
        assert S <= after - before <= S + 8 * MiB, (after - before, S)
        assert _used() - used0 <= S + 16 * MiB
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b)
        for h in ds.handles:
            ctx.release(h)
        ctx.trim()
        assert _held() - before == 0
        assert _used() - used0 <= 16 * MiB


def test_released_handles_return_hbm_c3():
    """configs[2] (C3, 10 000 odd buffers, 5.26 GB): restore re-creates them, then 90 %
    of the handles (in handle order) are released: about 90 % of the bytes return."""
    w = synth.c3_handle_stress()
    S = w.total_bytes
    with checl.Context() as ctx:
        tensors = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
        for t, b in zip(tensors, w.buffers):
            checl.debug_fill(t, w.seed, b.stream)
        torch.cuda.synchronize()
        handles = [ctx.register(t) for t in tensors]
        img = ctx.checkpoint_device(0, epoch=1)
        for h in handles:
            ctx.release(h)
        del tensors, t
        ctx.restore(img, 0)
        img.free()
        ctx.trim()
        full, full_used = _held(), _used()
        assert full >= S
        cut = int(len(handles) * 0.9)
        released = sum(b.size for b in w.buffers[:cut])
        for h in handles[:cut]:
            ctx.release(h)
        ctx.trim()
        dropped = full - _held()
        # every segment whose handles are all released went back (a segment is at most
        # 64 MiB: only the one holding the cut can stay)
        assert released - 64 * MiB <= dropped <= released + 64 * MiB, (dropped, released)
        assert full_used - _used() >= 0
        # the remaining handles still hold their bytes
        rng = np.random.default_rng(3)
        for i in rng.integers(cut, len(handles), 40):
            b = w.buffers[int(i)]
            got = ctx.tensor(handles[int(i)]).cpu().numpy()
            assert np.array_equal(got, synth.fill_bytes(b.size, w.seed, b.stream)), int(i)
        assert S > released


def test_restore_waits_for_work_pending_on_the_caller_stream():
    """The caching allocator hands restore a block the application freed while a kernel
    that writes it is still queued behind a long one; K2 must land after that write."""
    n = 8 * MiB
    with checl.Context() as ctx:
        ds = make_set(ctx, [n], seed=41)
        img = ctx.checkpoint_device(0, epoch=1)
        ctx.trim()
        torch.cuda.synchronize()
        x = torch.empty(n, dtype=torch.uint8, device=0)
        victim = x.data_ptr()
        torch.cuda._sleep(200_000_000)  # ~0.1 s of GPU time on the current stream
        x.fill_(0xAB)                  # queued behind it, writes the block
        del x                          # the block goes back to the cache (stream-ordered)
        rep = ctx.restore(img, 0, stream=torch.cuda.current_stream())
        assert rep.n_bad_chunks == 0
        ptr, nb, _ = ctx.translate(ds.handles[0])
        if ptr != victim:
            pytest.skip("the allocator did not hand out the freed block")
        torch.cuda.synchronize()
        assert np.array_equal(bound_bytes(ctx, ds.handles[0]), ds.host[0])
        img.free()


def test_release_during_checkpoint_is_deferred():
    sizes = [512 * MiB, 256 * MiB + 7, 700 * MiB + 1, 3 * MiB]
    with checl.Context() as ctx:
        ds = make_set(ctx, sizes, seed=51)
        img0 = ctx.checkpoint_device(0, epoch=1)
        ctx.restore(img0, 0)  # every buffer library-owned, one segment each
        img0.free()
        ctx.trim()
        ents = oracle_entries(ds)
        out, err = {}, []

        def run():
            try:
                out["img"] = ctx.checkpoint(0, epoch=2)  # pinned host image: ~30 ms over PCIe
            except Exception as e:  # pragma: no cover
                err.append(e)

        t = threading.Thread(target=run)
        t.start()
        time.sleep(0.004)
        ctx.release(ds.handles[2])  # while the checkpoint may be reading it
        junk = torch.full((sizes[2],), 0xCD, dtype=torch.uint8, device=0)  # would reuse a freed block
        t.join()
        assert not err, err
        got = out["img"].view()
        n_buf = int(out["img"].header()["n_buffers"])
        want = O.checkpoint(ents if n_buf == 4 else [e for i, e in enumerate(ents) if i != 2], device=0, epoch=2)
        assert np.array_equal(got, want)
        del junk
        out["img"].free()


def test_segment_boundaries_and_partial_release():
    """Segments (reading 18) around the 64 MiB cut: buffers just under, at and
    just over it, zero-size buffers between and at the ends, a segment made only of
    small buffers; every restore is bit-exact, the segment plan shows in the held bytes,
    and releasing every handle of one segment returns that segment alone."""
    sizes = [0, 64 * MiB - 1, 0, 64 * MiB, 3, 64 * MiB + 1, 5000, 7000, 0, 1, 32 * MiB, 33 * MiB, 0]
    with checl.Context() as ctx:
        ds = make_set(ctx, sizes, seed=61, offsets=[i % 4 for i in range(len(sizes))])
        img = ctx.checkpoint_device(0, epoch=1)
        for rep in range(3):  # a fresh allocation, then the spares of the previous commit
            ctx.restore(img, 0)
            for h, b in zip(ds.handles, ds.host):
                assert np.array_equal(bound_bytes(ctx, h), b), (rep, h)
        ctx.trim()
        held = _held()
        # the 33 MiB buffer would take the segment of the small buffers and the 32 MiB
        # one past 64 MiB, so a new segment starts with it (only the zero-size buffer
        # after it joins): releasing it returns that segment, ~33 MiB rounded up
        i = sizes.index(33 * MiB)
        ctx.release(ds.handles[i])
        ctx.trim()
        dropped = held - _held()
        assert 33 * MiB <= dropped <= 36 * MiB, dropped
        for h, b in zip(ds.handles[:i], ds.host[:i]):
            assert np.array_equal(bound_bytes(ctx, h), b), h
        img.free()
