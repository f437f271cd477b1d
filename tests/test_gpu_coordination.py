"""-m gpu: the global snapshot (§IV-B/C: "local snapshots are aggregated
into a global snapshot"; reading 16, a two-phase commit) on real images.

Two ranks share cuda:0 over gloo (one GPU here; the status all-reduce is the same
call as over NCCL). Each rank registers its own buffers and calls
coordination.coordinated_checkpoint three ways: a new host image, into= a reused
image, and on_device=True (HBM image). Commit path: each rank's image equals the
oracle's image of that rank's registry byte for byte. Abort path: rank 1's local
checkpoint fails for real: its context is BUSY, held by a restore that is blocked
inside the context's allocator callback. Every rank must then drop the snapshot: a
new image is freed, an into= image survives (not freed, not returned), and with an
ImagePair the last committed global snapshot survives unchanged.
"""
import os
import socket

import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import ctypes as C
    import threading

    import numpy as np
    import torch
    import torch.distributed as dist

    from oracle import oracle as O
    from paper_conf_ipps_takizawakskk11_b200 import checl
    from paper_conf_ipps_takizawakskk11_b200.coordination import ImagePair, coordinated_checkpoint
    from tests.gpu_util import make_set, oracle_entries

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    res = {}
    try:
        # an allocator that can be made to block: the restore holding the context busy
        arm, entered, gate = threading.Event(), threading.Event(), threading.Event()

        @C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)
        def _alloc(nbytes, device, stream, user):
            if arm.is_set():
                entered.set()
                gate.wait(60)
            return torch.cuda.caching_allocator_alloc(int(nbytes), device, int(stream or 0))

        @C.CFUNCTYPE(None, C.c_void_p, C.c_int, C.c_void_p, C.c_void_p)
        def _free(ptr, device, stream, user):
            torch.cuda.caching_allocator_delete(int(ptr))

        ctx = checl.Context(allocator=checl.Allocator(_alloc, _free, None))
        sizes = [1 << 20, 65536 * 3 + 17 + rank, 0, 4097, 300007 + 64 * rank]
        ds = make_set(ctx, sizes, seed=200 + rank)
        want = lambda epoch: O.checkpoint(oracle_entries(ds), device=0, epoch=epoch)  # noqa: E731
        base_img = ctx.checkpoint(0, epoch=1)

        made = []

        class Recorder:  # the context, recording the images the local checkpoints return
            def count(self, d):
                return ctx.count(d)

            def checkpoint(self, *a, **k):
                im = ctx.checkpoint(*a, **k)
                made.append(im)
                return im

            def checkpoint_device(self, *a, **k):
                im = ctx.checkpoint_device(*a, **k)
                made.append(im)
                return im

        rc = Recorder()

        def voted(fn, fail):
            """fn() on every rank; with fail, rank 1's context is busy meanwhile."""
            if not (fail and rank == 1):
                return fn()
            ctx.trim()  # (no spare segment: the restore must call the allocator)
            arm.set()
            t = threading.Thread(target=lambda: ctx.restore(base_img, 0))
            t.start()
            assert entered.wait(60), "restore did not reach the allocator"
            try:
                return fn()
            finally:
                arm.clear()
                gate.set()
                t.join(60)
                entered.clear()
                gate.clear()

        # -- commit path
        s = coordinated_checkpoint(rc, 0, epoch=5)
        res["host_commit"] = s.committed and np.array_equal(s.image.view(), want(5))
        s.image.free()
        reuse = ctx.checkpoint(0, epoch=2)
        s = coordinated_checkpoint(rc, 0, epoch=6, into=reuse)
        res["into_commit"] = s.committed and s.image is reuse and np.array_equal(reuse.view(), want(6))
        s = coordinated_checkpoint(rc, 0, epoch=7, on_device=True)
        h = s.image.to_host()
        res["device_commit"] = s.committed and np.array_equal(h.view(), want(7))
        h.free()
        s.image.free()

        # -- abort path: rank 1 BUSY
        made.clear()
        s = voted(lambda: coordinated_checkpoint(rc, 0, epoch=8), True)
        res["host_abort"] = (not s.committed and s.image is None and s.failures == 1 and
                             all(not im._p for im in made))  # the local image rank 0 made was freed
        made.clear()
        s = voted(lambda: coordinated_checkpoint(rc, 0, epoch=9, on_device=True), True)
        res["device_abort"] = not s.committed and s.image is None and all(not im._p for im in made)
        s = voted(lambda: coordinated_checkpoint(rc, 0, epoch=10, into=reuse), True)
        res["into_abort"] = (not s.committed and s.image is None and bool(reuse._p) and
                             reuse.view().size == want(6).size)
        pair = ImagePair()
        s1 = voted(lambda: coordinated_checkpoint(ctx, 0, epoch=11, into=pair), False)
        s2 = voted(lambda: coordinated_checkpoint(ctx, 0, epoch=12, into=pair), True)
        kept = np.array_equal(pair.committed.view(), want(11))  # the abort left epoch 11 intact
        s3 = voted(lambda: coordinated_checkpoint(ctx, 0, epoch=13, into=pair), False)
        res["pair"] = (s1.committed and not s2.committed and s3.committed and kept and
                       np.array_equal(pair.committed.view(), want(13)))
        pair.free()
        reuse.free()
        base_img.free()
        ctx.close()
    except Exception as e:  # report instead of hanging the other rank
        res["error"] = repr(e)
    q.put((rank, res))
    dist.destroy_process_group()


def test_coordinated_checkpoint_real_images_commit_and_abort():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=600) for _ in range(2))
    for p in ps:
        p.join(timeout=120)
    for rank, res in out:
        assert "error" not in res, (rank, res)
        for k in ("host_commit", "into_commit", "device_commit", "host_abort", "device_abort", "into_abort",
                  "pair"):
            assert res.get(k), (rank, k, res)


def _nccl_worker(port, q):
    import numpy as np
    import torch
    import torch.distributed as dist

    from oracle import oracle as O
    from paper_conf_ipps_takizawakskk11_b200 import checl
    from paper_conf_ipps_takizawakskk11_b200.coordination import agree, coordinated, coordinated_checkpoint
    from tests.gpu_util import make_set, oracle_entries

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    res = {}
    try:
        res["backend"] = dist.get_backend()
        # the status vector on the GPU through NCCL: world 1 returns the inputs
        res["agree"] = agree(False, 7, 12345, (3 << 48) | 77, device=0) == (0, 7, 12345, True, (3 << 48) | 77)
        ctx = checl.Context()
        ds = make_set(ctx, [1 << 20, 65537, 0, 4097], seed=9)
        for on_device in (False, True):
            snap = coordinated_checkpoint(ctx, 0, epoch=5, on_device=on_device)
            want = O.checkpoint(oracle_entries(ds), device=0, epoch=5)
            got = snap.image.to_host().view() if on_device else snap.image.view()
            res[f"commit_{on_device}"] = snap.committed and np.array_equal(got, want)
            snap.image.free()

        def failing():
            raise RuntimeError("local snapshot failed")

        snap = coordinated(failing, epoch=6, device=0)
        res["abort"] = (not snap.committed) and snap.image is None and snap.failures == 1
        ctx.close()
    except Exception as e:
        res["error"] = repr(e)
    q.put(res)
    dist.destroy_process_group()


def test_status_allreduce_over_nccl_world1():
    """The coordination all-reduce as it runs on a GPU box: NCCL backend, the status
    vector in HBM (one rank: NCCL refuses two ranks on one GPU). Commit with a host
    and an HBM image equal to the oracle's; a failed local snapshot aborts."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_nccl_worker, args=(_free_port(), q))
    p.start()
    res = q.get(timeout=600)
    p.join(timeout=120)
    assert "error" not in res, res
    assert res["backend"] == "nccl"
    for k in ("agree", "commit_False", "commit_True", "abort"):
        assert res.get(k), (k, res)
