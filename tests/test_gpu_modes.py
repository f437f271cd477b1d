"""-m gpu: the delayed checkpointing mode (§III-C)
and the writing phase (row 4; L16 step 3, Table I) through the C ABI, bit-exact
against the oracle."""
import os
import signal

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


@pytest.fixture()
def ctx():
    c = checl.Context()
    yield c
    c.close()


def test_delayed_mode_checkpoints_at_the_sync_point(ctx):
    ds = make_set(ctx, [1 << 20, 70001, 0, 5], seed=12)
    s = torch.cuda.Stream(DEV)
    # the application's queued work (not on registered buffers) keeps the stream busy
    a = torch.randn(4096, 4096, device=DEV)
    with torch.cuda.stream(s):
        for _ in range(20):
            a = a @ a
            a = a / a.norm()
    assert ctx.sync_point(DEV, s, epoch=1) is None  # nothing requested: only the clFinish
    ctx.install_signal(signal.SIGUSR1)
    os.kill(os.getpid(), signal.SIGUSR1)
    assert ctx.checkpoint_pending()
    with torch.cuda.stream(s):
        for _ in range(20):
            a = a @ a
            a = a / a.norm()
    img = ctx.sync_point(DEV, s, epoch=2)
    assert img is not None and not ctx.checkpoint_pending()
    t = ctx.last_timing()
    assert t["sync_ms"] < 5.0  # the stream was already drained by the sync point
    want = O.checkpoint(oracle_entries(ds), device=DEV, epoch=2)
    assert np.array_equal(img.view(), want)
    # reuse of an image at the next request
    ctx.request_checkpoint()
    again = ctx.sync_point(DEV, None, epoch=3, into=img)
    assert again is img
    assert np.array_equal(img.view(), O.checkpoint(oracle_entries(ds), device=DEV, epoch=3))
    checl.lib.checl_install_signal(None, signal.SIGUSR1)
    release_all(ctx, ds)


@pytest.mark.parametrize("where", ["device", "host"])
def test_image_file_round_trip_and_restore(ctx, tmp_path, where):
    ds = make_set(ctx, [300007, 65536, 17, 1 << 20], seed=13, offsets=[0, 4, 1, 0])
    want = O.checkpoint(oracle_entries(ds), device=DEV, epoch=4)
    img = ctx.checkpoint_device(DEV, epoch=4) if where == "device" else ctx.checkpoint(DEV, epoch=4)
    path = str(tmp_path / "snap.checl")
    img.write(path, direct=True, sync=True)
    assert os.path.getsize(path) == want.size
    back = checl.Image.read(path)
    assert np.array_equal(back.view(), want)
    for t in ds.tensors:
        t.zero_()
    rep = ctx.restore(back, DEV)
    assert rep.n_bad_chunks == 0
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)
    # a bit flipped on disk is caught at restore and localised like the oracle's
    raw = bytearray(open(path, "rb").read())
    poff = int(back.header()["payload_off"])
    raw[poff + 70000] ^= 4
    open(path, "wb").write(bytes(raw))
    bad = checl.Image.read(path, direct=False)
    with pytest.raises(checl.CheclError) as ei:
        ctx.restore(bad, DEV)
    st, rep_o, _ = O.restore(np.frombuffer(bytes(raw), np.uint8))
    assert ei.value.status == checl.ERR_CRC_MISMATCH and st == O.CRC_MISMATCH
    assert ei.value.report.first_bad_chunk == rep_o["first_bad_chunk"]


def test_pinned_pool_reuses_freed_images(ctx):
    ds = make_set(ctx, [8 << 20], seed=14)
    F = ctx.checkpoint(DEV, epoch=0)
    base = F
    for e in range(1, 6):
        ds.tensors[0][e * 65536:e * 65536 + 1].add_(1)
        ds.host[0][e * 65536] += 1
        d = ctx.checkpoint_incremental(DEV, base, epoch=e)
        if base is not F:
            base.free()
        base = d
        t = ctx.last_timing()
        assert d.header()["n_present"] == 1
    assert t["total_ms"] < 20.0
    release_all(ctx, ds)
