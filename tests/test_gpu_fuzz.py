"""-m gpu: seeded random registries through the C ABI against the oracle.

Each case draws a registry (1-40 buffers, sizes 0 B - 1.2 MB with a heavy tail of
tiny and odd sizes, source misalignments 0-15 B, handle order shuffled by
release/re-register), a staging configuration (one launch in HBM, or small slots
that split buffers across stages), then checks: the host image equals the oracle's
byte for byte, the HBM image's metadata mirror equals it too, restore from both
reproduces every buffer, a random single-bit payload flip is reported at the
oracle's chunk, and an incremental image after random rewrites equals the
oracle's delta (exact rule on even cases, CRC rule on odd ones)."""
import os

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


def _sizes(rng, n):
    out = []
    for _ in range(n):
        u = rng.random()
        if u < 0.1:
            out.append(0)
        elif u < 0.35:
            out.append(int(rng.integers(1, 300)))
        elif u < 0.8:
            out.append(int(rng.integers(300, 200_000)))
        else:
            out.append(int(rng.integers(200_000, 1_200_000)))
    return out


# CHECL_FUZZ_CASES widens the sweep (default 24 cases; profiles/ records a 400-case run)
@pytest.mark.parametrize("case", range(int(os.environ.get("CHECL_FUZZ_CASES", "24"))))
def test_random_registry(case):
    rng = np.random.default_rng(1000 + case)
    ctx = checl.Context()
    if case % 3 == 1:
        ctx.set_staging(65536 * int(rng.integers(2, 6)), int(rng.integers(1, 4)))
    n = int(rng.integers(1, 41))
    sizes = _sizes(rng, n)
    offs = [int(rng.integers(0, 16)) for _ in range(n)]
    ds = make_set(ctx, sizes, seed=case, offsets=offs, kind=int(rng.integers(0, 3)))
    # shuffle database order: release and re-register a random subset (new, larger ids)
    for i in rng.choice(n, size=n // 3, replace=False):
        ctx.release(ds.handles[i])
        ds.handles[i] = ctx.register(ds.tensors[i], ds.flags[i])
    epoch = int(rng.integers(0, 1 << 40))
    want = O.checkpoint(oracle_entries(ds), device=DEV, epoch=epoch)
    img = ctx.checkpoint(DEV, epoch=epoch)
    assert np.array_equal(img.view(), want)
    dimg = ctx.checkpoint_device(DEV, epoch=epoch)
    assert np.array_equal(dimg.view(), want[:dimg.view().size])
    for im in (img, dimg):
        rep = ctx.restore(im, DEV)
        assert rep.n_bad_chunks == 0
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b)
    # one random payload bit flipped: the oracle's chunk, nothing rebound
    poff = int(img.header()["payload_off"])
    if want.size > poff:
        pos = int(rng.integers(poff, want.size))
        bad = want.copy()
        bad[pos] ^= 1 << int(rng.integers(0, 8))
        st, rep_o, _ = O.restore(bad)
        before = [ctx.translate(h) for h in ds.handles]
        with pytest.raises(checl.CheclError) as ei:
            ctx.restore(checl.Image.wrap(bad), DEV)
        assert st == O.CRC_MISMATCH and ei.value.status == checl.ERR_CRC_MISMATCH
        assert ei.value.report.first_bad_chunk == rep_o["first_bad_chunk"]
        assert [ctx.translate(h) for h in ds.handles] == before
    # incremental after random rewrites of the live (restored) buffers
    live = [ctx.tensor(h) if b.size else None for h, b in zip(ds.handles, ds.host)]
    for _ in range(int(rng.integers(0, 6))):
        i = int(rng.integers(0, n))
        if ds.host[i].size:
            p = int(rng.integers(0, ds.host[i].size))
            live[i][p:p + 1].bitwise_xor_(0x21)
            ds.host[i][p] ^= 0x21
    torch.cuda.synchronize()
    if case % 2:  # the CRC rule (reading 21)
        d = ctx.checkpoint_incremental(DEV, img, epoch=epoch + 1, rule=checl.DIRTY_CRC)
        want_d = O.checkpoint_incremental(oracle_entries(ds), want, device=DEV, epoch=epoch + 1)
    else:  # the exact rule (default; reading 25): the base's state is the full image `want`
        d = ctx.checkpoint_incremental(DEV, img, epoch=epoch + 1)
        want_d = O.checkpoint_incremental(oracle_entries(ds), want, device=DEV, epoch=epoch + 1, rule=O.RULE_BYTES,
                                          base_full=want)
    assert np.array_equal(d.view(), want_d)
    release_all(ctx, ds)
    ctx.close()
