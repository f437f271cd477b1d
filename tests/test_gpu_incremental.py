"""-m gpu: incremental checkpoint (§IV-D) through
the C ABI against the CPU oracle, bit-exact: delta images equal the oracle's
byte for byte (present bitmap, CRC table, compacted payload), chains restore to
the exact bytes, the library's merge equals the oracle's, corruption in a delta
is localised like the oracle's and nothing is rebound."""
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


def _mutate(ds, changes):
    """XOR byte values into the registered device views and the host copies."""
    for i, pos, x in changes:
        ds.tensors[i][pos:pos + 1].bitwise_xor_(x)
        ds.host[i][pos] ^= x
    torch.cuda.synchronize()


def _eq(got, want, what):
    assert got.size == want.size, (what, got.size, want.size)
    if not np.array_equal(got, want):
        bad = np.nonzero(got != want)[0]
        raise AssertionError(f"{what}: differs at {bad.size} bytes, first {bad[:8]}")


def _random_changes(ds, rng, n):
    idx = [i for i, h in enumerate(ds.host) if h.size]
    return [(int(i), int(rng.integers(0, ds.host[i].size)), int(rng.integers(1, 256)))
            for i in rng.choice(idx, size=n)]


@pytest.mark.parametrize("slot", [None, 131072, 196608])
def test_delta_images_equal_oracle(ctx, slot):
    if slot:
        ctx.set_staging(slot, 2)
    rng = np.random.default_rng(31)
    sizes = [300007, 0, 65536, 65537, 17, 1 << 20, 131072 + 255]
    ds = make_set(ctx, sizes, seed=4, offsets=[0, 0, 1, 4, 0, 8, 3])
    F = ctx.checkpoint(DEV, epoch=1)
    base_o = O.checkpoint(oracle_entries(ds), device=DEV, epoch=1)
    _eq(F.view(), base_o, "base")
    prev_g, prev_o = F, base_o
    for step, nchg in enumerate([0, 1, 5, 40]):
        _mutate(ds, _random_changes(ds, rng, nchg))
        D = ctx.checkpoint_incremental(DEV, prev_g, epoch=2 + step)
        want = O.checkpoint_incremental(oracle_entries(ds), prev_o, device=DEV, epoch=2 + step)
        _eq(D.view(), want, f"delta {step}")
        assert D.header()["flags"] == 1
        prev_g, prev_o = D, want
    # everything changed: the compacted payload is the full payload
    for i, h in enumerate(ds.host):
        if h.size:
            ds.tensors[i].bitwise_not_()
            ds.host[i] = ~h
    torch.cuda.synchronize()
    D = ctx.checkpoint_incremental(DEV, prev_g, epoch=9)
    want = O.checkpoint_incremental(oracle_entries(ds), prev_o, device=DEV, epoch=9)
    _eq(D.view(), want, "all changed")
    assert D.header()["n_present"] == D.header()["n_chunks"]


def test_device_image_as_base(ctx):
    ds = make_set(ctx, [200000, 4097], seed=5)
    Fd = ctx.checkpoint_device(DEV, epoch=1)
    base_o = O.checkpoint(oracle_entries(ds), device=DEV, epoch=1)
    _mutate(ds, [(0, 123456, 7)])
    D = ctx.checkpoint_incremental(DEV, Fd, epoch=2)
    _eq(D.view(), O.checkpoint_incremental(oracle_entries(ds), base_o, device=DEV, epoch=2), "delta on HBM base")


def test_layout_change_gives_full_image(ctx):
    ds = make_set(ctx, [5000, 70000], seed=6)
    F = ctx.checkpoint(DEV, epoch=1)
    extra = torch.full((33,), 7, dtype=torch.uint8, device=DEV)
    h = ctx.register(extra, 9)
    ents = oracle_entries(ds) + [O.Entry(h, extra.cpu().numpy(), 9)]
    D = ctx.checkpoint_incremental(DEV, F, epoch=2)
    _eq(D.view(), O.checkpoint(ents, device=DEV, epoch=2), "layout change -> full")
    assert D.header()["flags"] == 0


def test_restore_chain_and_merge(ctx):
    rng = np.random.default_rng(32)
    ds = make_set(ctx, [400001, 3, 65536 * 3, 0, 9999], seed=7, offsets=[0, 1, 0, 0, 4])
    chain = [ctx.checkpoint(DEV, epoch=0)]
    chain_o = [O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)]
    for e in range(1, 4):
        _mutate(ds, _random_changes(ds, rng, 3 * e))
        chain.append(ctx.checkpoint_incremental(DEV, chain[-1], epoch=e))
        chain_o.append(O.checkpoint_incremental(oracle_entries(ds), chain_o[-1], device=DEV, epoch=e))
    final = [h.copy() for h in ds.host]
    # library merge == oracle merge == the full checkpoint of the final state
    M = chain[0]
    Mo = chain_o[0]
    for d, do in zip(chain[1:], chain_o[1:]):
        M = M.merge(d)
        st, Mo = O.merge(Mo, do)
        assert st == 0
        _eq(M.view(), Mo, "merge")
    _eq(M.view(), O.checkpoint(oracle_entries(ds), device=DEV, epoch=3), "merge == full")
    # scribble over the live buffers, then restore the chain
    for t in ds.tensors:
        t.zero_()
    torch.cuda.synchronize()
    rep = ctx.restore_chain(chain, DEV)
    st, rep_o, _ = O.restore_chain(chain_o)
    assert st == 0 and rep.n_bad_chunks == 0 and rep.n_chunks == rep_o["n_chunks"]
    assert rep.payload_bytes == rep_o["payload_bytes"]
    for h, want in zip(ds.handles, final):
        assert np.array_equal(bound_bytes(ctx, h), want)
    release_all(ctx, ds)


def test_restore_chain_corruption_localised_and_nothing_rebound(ctx):
    ds = make_set(ctx, [300000, 70000], seed=8)
    F = ctx.checkpoint(DEV, epoch=0)
    Fo = O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)
    _mutate(ds, [(0, 200000, 3), (1, 69999, 1)])
    D = ctx.checkpoint_incremental(DEV, F, epoch=1)
    Do = O.checkpoint_incremental(oracle_entries(ds), Fo, device=DEV, epoch=1)
    h = D.header()
    bound_before = [ctx.translate(x) for x in ds.handles]
    for pos in (h["payload_off"] + 5, h["image_bytes"] - 1):
        D.corrupt(pos, 0x20)
        bad_o = Do.copy()
        bad_o[pos] ^= 0x20
        with pytest.raises(checl.CheclError) as ei:
            ctx.restore_chain([F, D], DEV)
        assert ei.value.status == checl.ERR_CRC_MISMATCH
        st, rep_o, _ = O.restore_chain([Fo, bad_o])
        assert st == O.CRC_MISMATCH
        r = ei.value.report
        assert (r.n_bad_chunks, r.first_bad_chunk, r.first_bad_handle) == (
            rep_o["n_bad_chunks"], rep_o["first_bad_chunk"], rep_o["first_bad_handle"])
        assert [ctx.translate(x) for x in ds.handles] == bound_before
        D.corrupt(pos, 0x20)
    # metadata corruption / broken links / a delta alone
    D.corrupt(100, 1)
    with pytest.raises(checl.CheclError) as ei:
        ctx.restore_chain([F, D], DEV)
    assert ei.value.status == checl.ERR_BAD_IMAGE
    D.corrupt(100, 1)
    with pytest.raises(checl.CheclError) as ei:
        ctx.restore(D, DEV)
    assert ei.value.status == checl.ERR_BAD_IMAGE
    with pytest.raises(checl.CheclError) as ei:
        ctx.restore_chain([D, F], DEV)
    assert ei.value.status == checl.ERR_BAD_IMAGE
    release_all(ctx, ds)


def test_c2_full_size_incremental_ten_percent(ctx):
    """configs[1] (SDK mix, 463 MB) with ~10% of its chunks rewritten between epochs."""
    import synth
    w = synth.c2_sdk_mix()
    sizes = [b.size for b in w.buffers]
    ds = make_set(ctx, sizes, seed=w.seed)
    F = ctx.checkpoint(DEV, epoch=0)
    Fo = O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)
    rng = np.random.default_rng(33)
    nch = F.header()["n_chunks"]
    _mutate(ds, _random_changes(ds, rng, nch // 10))
    D = ctx.checkpoint_incremental(DEV, F, epoch=1)
    Do = O.checkpoint_incremental(oracle_entries(ds), Fo, device=DEV, epoch=1)
    _eq(D.view(), Do, "C2 delta")
    rep = ctx.restore_chain([F, D], DEV)
    assert rep.n_bad_chunks == 0
    for i in rng.choice(len(sizes), 4, replace=False):
        assert np.array_equal(bound_bytes(ctx, ds.handles[i]), ds.host[i])
    release_all(ctx, ds)
