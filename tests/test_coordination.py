"""-m "not gpu": the coordinated (global) snapshot protocol over torch.distributed
gloo on CPU, world_size 2 and 8. Local snapshots are mocked;
the commit rule is PAPER.md L40's global snapshot read as a two-phase commit
(reading 16): commit iff no rank failed and all epochs agree."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class FakeImage:
    def __init__(self):
        self.freed = False

    def free(self):
        self.freed = True


def _worker(rank, world, port, scenario, q):
    import torch.distributed as dist
    from paper_conf_ipps_takizawakskk11_b200.coordination import coordinated
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    img = FakeImage()

    def local():
        if scenario in ("fail", "fail_keep") and rank == world - 1:
            raise RuntimeError("injected local checkpoint failure")
        return img, 3 + rank, 1000 * (rank + 1)

    epoch = 7 if not (scenario == "epoch" and rank == 0) else 8
    if scenario == "epoch_hi":  # differ only in the top 16 bits
        epoch = 7 + ((1 << 48) if rank == 1 else 0)
    if scenario == "epoch_big":  # equal, all 64 bits in use
        epoch = (1 << 63) - 3
    g = coordinated(local, epoch, keep=img if scenario == "fail_keep" else None)
    q.put((rank, g.committed, g.failures, g.n_buffers, g.total_bytes, g.epochs_agree, img.freed, g.image is None))
    dist.destroy_process_group()


def _run(world, scenario):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, scenario, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out)


@pytest.mark.parametrize("world", [2, 8])
def test_commit_sums_closed_form(world):
    for rank, ok, f, nb, tb, same, freed, none in _run(world, "ok"):
        assert ok and f == 0 and same and not freed and not none
        assert nb == sum(3 + r for r in range(world))           # closed form of the SUM
        assert tb == sum(1000 * (r + 1) for r in range(world))


@pytest.mark.parametrize("world", [2, 8])
def test_one_failing_rank_aborts_everyone(world):
    res = _run(world, "fail")
    for rank, ok, f, nb, tb, same, freed, none in res:
        assert not ok and f == 1 and none
        if rank != world - 1:
            assert freed  # surviving ranks free their local images


def test_epoch_disagreement_aborts():
    for rank, ok, f, nb, tb, same, freed, none in _run(2, "epoch"):
        assert not ok and f == 0 and not same and none


def test_epoch_agreement_exact_in_every_16_bit_part():
    for rank, ok, f, nb, tb, same, freed, none in _run(3, "epoch_hi"):
        assert not ok and not same and none
    for rank, ok, f, nb, tb, same, freed, none in _run(3, "epoch_big"):
        assert ok and same and not none


def test_abort_keeps_caller_owned_reused_image():
    """An image passed for reuse (checl_checkpoint_into) stays the caller's on abort:
    not freed, not returned, committed = False."""
    for rank, ok, f, nb, tb, same, freed, none in _run(2, "fail_keep"):
        assert not ok and f == 1 and none and not freed


class FakeCtx:
    """Stands in for checl.Context in coordinated_checkpoint: count() and
    checkpoint(device, stream, epoch, into=None) (a new image or the reused one,
    stamped with the epoch). Rank `fail_rank` fails its local checkpoint at the epochs
    listed in `fail_at`."""

    def __init__(self, rank, fail_rank, fail_at):
        self.rank, self.fail_rank, self.fail_at = rank, fail_rank, fail_at
        self.made = []

    def count(self, device):
        return 2, 64

    def checkpoint(self, device, stream=None, epoch=0, into=None):
        if self.rank == self.fail_rank and epoch in self.fail_at:
            raise RuntimeError("local checkpoint failed")
        img = into if into is not None else FakeImage()
        if into is None:
            self.made.append(img)
        img.epoch = epoch
        return img


def _pair_worker(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_ipps_takizawakskk11_b200.coordination import ImagePair, coordinated_checkpoint
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ctx = FakeCtx(rank, world - 1, {2, 3, 5})
    pair = ImagePair()
    log = []
    for epoch in range(1, 7):
        snap = coordinated_checkpoint(ctx, 0, epoch, into=pair)
        c = pair.committed
        log.append((epoch, snap.committed, c.epoch if c is not None else None, c.freed if c is not None else None))
    q.put((rank, log, len(ctx.made)))
    dist.destroy_process_group()


def test_image_pair_keeps_last_committed_snapshot_on_abort():
    """Double-buffered global snapshots (reading 16): every new
    local snapshot goes into the image that does not hold the last committed one, so
    after an aborted vote the committed image still holds the previous global
    snapshot (epochs 2, 3 and 5 abort here: rank 1 fails), and only two images are
    ever pinned per rank."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_pair_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=120) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    want = [(1, True, 1, False), (2, False, 1, False), (3, False, 1, False), (4, True, 4, False),
            (5, False, 4, False), (6, True, 6, False)]
    for rank, log, made in out:
        assert log == want, (rank, log)
        assert made <= 2 + (2 if rank == 0 else 0), made  # rank 0's aborted first-slot image is freed and re-made
