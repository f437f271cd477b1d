"""-m gpu: incremental checkpoint (§IV-D) through
the C ABI against the CPU oracle, bit-exact: delta images equal the oracle's
byte for byte (present bitmap, CRC table, compacted payload), chains restore to
the exact bytes, the library's merge equals the oracle's, corruption in a delta
is localised like the oracle's and nothing is rebound. Both dirty rules (FORMAT.md
"Present set"): bytes (default, exact; reading 25 — the oracle gets the
full image of the base's state) and CRC (reading 21)."""
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


RULES = [checl.DIRTY_BYTES, checl.DIRTY_CRC]


def _odelta(ds, base_o, base_full_o, epoch, rule):
    """The oracle's delta of ds's current state against base_o (base_full_o = the
    full image of base_o's state, for the bytes rule)."""
    if rule == checl.DIRTY_BYTES:
        return O.checkpoint_incremental(oracle_entries(ds), base_o, device=DEV, epoch=epoch, rule=O.RULE_BYTES,
                                        base_full=base_full_o)
    return O.checkpoint_incremental(oracle_entries(ds), base_o, device=DEV, epoch=epoch)


def _random_changes(ds, rng, n):
    idx = [i for i, h in enumerate(ds.host) if h.size]
    return [(int(i), int(rng.integers(0, ds.host[i].size)), int(rng.integers(1, 256)))
            for i in rng.choice(idx, size=n)]


@pytest.mark.parametrize("rule", RULES)
@pytest.mark.parametrize("slot", [None, 131072, 196608])
def test_delta_images_equal_oracle(ctx, slot, rule):
    if slot:
        ctx.set_staging(slot, 2)
    rng = np.random.default_rng(31)
    sizes = [300007, 0, 65536, 65537, 17, 1 << 20, 131072 + 255]
    ds = make_set(ctx, sizes, seed=4, offsets=[0, 0, 1, 4, 0, 8, 3])
    F = ctx.checkpoint(DEV, epoch=1)
    base_o = O.checkpoint(oracle_entries(ds), device=DEV, epoch=1)
    _eq(F.view(), base_o, "base")
    prev_g, prev_o, prev_full = F, base_o, base_o
    for step, nchg in enumerate([0, 1, 5, 40]):
        _mutate(ds, _random_changes(ds, rng, nchg))
        D = ctx.checkpoint_incremental(DEV, prev_g, epoch=2 + step, rule=rule)
        want = _odelta(ds, prev_o, prev_full, 2 + step, rule)
        _eq(D.view(), want, f"delta {step}")
        assert D.header()["flags"] == 1 and D.header()["dirty_rule"] == rule
        prev_g, prev_o, prev_full = D, want, O.checkpoint(oracle_entries(ds), device=DEV, epoch=2 + step)
    # everything changed: the compacted payload is the full payload
    for i, h in enumerate(ds.host):
        if h.size:
            ds.tensors[i].bitwise_not_()
            ds.host[i] = ~h
    torch.cuda.synchronize()
    D = ctx.checkpoint_incremental(DEV, prev_g, epoch=9, rule=rule)
    want = _odelta(ds, prev_o, prev_full, 9, rule)
    _eq(D.view(), want, "all changed")
    assert D.header()["n_present"] == D.header()["n_chunks"]


@pytest.mark.parametrize("rule", RULES)
def test_device_image_as_base(ctx, rule):
    ds = make_set(ctx, [200000, 4097], seed=5)
    Fd = ctx.checkpoint_device(DEV, epoch=1)
    base_o = O.checkpoint(oracle_entries(ds), device=DEV, epoch=1)
    _mutate(ds, [(0, 123456, 7)])
    D = ctx.checkpoint_incremental(DEV, Fd, epoch=2, rule=rule)
    _eq(D.view(), _odelta(ds, base_o, base_o, 2, rule), "delta on HBM base")


@pytest.mark.parametrize("rule", RULES)
def test_layout_change_gives_full_image(ctx, rule):
    ds = make_set(ctx, [5000, 70000], seed=6)
    F = ctx.checkpoint(DEV, epoch=1)
    extra = torch.full((33,), 7, dtype=torch.uint8, device=DEV)
    h = ctx.register(extra, 9)
    ents = oracle_entries(ds) + [O.Entry(h, extra.cpu().numpy(), 9)]
    D = ctx.checkpoint_incremental(DEV, F, epoch=2, rule=rule)
    _eq(D.view(), O.checkpoint(ents, device=DEV, epoch=2), "layout change -> full")
    assert D.header()["flags"] == 0


@pytest.mark.parametrize("rule", RULES)
def test_restore_chain_and_merge(ctx, rule):
    rng = np.random.default_rng(32)
    ds = make_set(ctx, [400001, 3, 65536 * 3, 0, 9999], seed=7, offsets=[0, 1, 0, 0, 4])
    chain = [ctx.checkpoint(DEV, epoch=0)]
    chain_o = [O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)]
    full_o = chain_o[0]
    for e in range(1, 4):
        _mutate(ds, _random_changes(ds, rng, 3 * e))
        chain.append(ctx.checkpoint_incremental(DEV, chain[-1], epoch=e, rule=rule))
        chain_o.append(_odelta(ds, chain_o[-1], full_o, e, rule))
        full_o = O.checkpoint(oracle_entries(ds), device=DEV, epoch=e)
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


@pytest.mark.parametrize("rule", RULES)
def test_restore_chain_corruption_localised_and_nothing_rebound(ctx, rule):
    ds = make_set(ctx, [300000, 70000], seed=8)
    F = ctx.checkpoint(DEV, epoch=0)
    Fo = O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)
    _mutate(ds, [(0, 200000, 3), (1, 69999, 1)])
    D = ctx.checkpoint_incremental(DEV, F, epoch=1, rule=rule)
    Do = _odelta(ds, Fo, Fo, 1, rule)
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


@pytest.mark.parametrize("rule", RULES)
def test_c2_full_size_incremental_ten_percent(ctx, rule):
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
    D = ctx.checkpoint_incremental(DEV, F, epoch=1, rule=rule)
    Do = _odelta(ds, Fo, Fo, 1, rule)
    _eq(D.view(), Do, "C2 delta")
    rep = ctx.restore_chain([F, D], DEV)
    assert rep.n_bad_chunks == 0
    for i in rng.choice(len(sizes), 4, replace=False):
        assert np.array_equal(bound_bytes(ctx, ds.handles[i]), ds.host[i])
    release_all(ctx, ds)


def _crc_blind(n=64):
    """A change vector whose CRC32C difference is zero (GF(2) elimination, as in
    tests/test_oracle_incremental.py)."""
    base = np.zeros(n, np.uint8)
    c0 = O.crc32c(base)
    pivots, combo = {}, None
    for i in range(40):
        e = base.copy()
        e[i // 8] ^= 1 << (i % 8)
        v, mask = O.crc32c(e) ^ c0, 1 << i
        while v:
            hb = v.bit_length() - 1
            if hb not in pivots:
                pivots[hb] = (v, mask)
                break
            pv, pm = pivots[hb]
            v ^= pv
            mask ^= pm
        if v == 0:
            combo = mask
            break
    return [(i // 8, 1 << (i % 8)) for i in range(40) if combo >> i & 1]


def test_crc_blind_change_exact_rule_writes_it(ctx):
    """A change the CRC cannot see: the default (bytes) rule writes its chunk and the
    chain restores the new bytes; the CRC rule leaves it out, like the oracle."""
    ds = make_set(ctx, [200000, 70001], seed=9)
    F = ctx.checkpoint(DEV, epoch=0)
    Fo = O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)
    flips = [(0, 65536 * 2 + 100 + pos, x) for pos, x in _crc_blind()]
    _mutate(ds, flips)
    assert O.crc32c(ds.host[0][65536 * 2:65536 * 3]) == O.crc32c(
        np.frombuffer(F.view(), np.uint8)[F.header()["payload_off"] + 65536 * 2:][:65536])
    Dc = ctx.checkpoint_incremental(DEV, F, epoch=1, rule=checl.DIRTY_CRC)
    _eq(Dc.view(), _odelta(ds, Fo, Fo, 1, checl.DIRTY_CRC), "CRC rule")
    assert Dc.header()["n_present"] == 0
    D = ctx.checkpoint_incremental(DEV, F, epoch=1)
    _eq(D.view(), _odelta(ds, Fo, Fo, 1, checl.DIRTY_BYTES), "bytes rule")
    assert D.header()["n_present"] == 1 and D.header()["dirty_rule"] == 1
    _eq(F.merge(D).view(), O.checkpoint(oracle_entries(ds), device=DEV, epoch=1), "merge == full")
    for t in ds.tensors:
        t.zero_()
    torch.cuda.synchronize()
    ctx.restore_chain([F, D], DEV)
    for h, want in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), want)
    release_all(ctx, ds)


def test_exact_rule_shadow_follows_the_chain_and_reseeds(ctx):
    """The device copy of the base state (the shadow) follows a chain of deltas; a
    delta taken against an older base (whose state the device no longer holds) is the
    full image, and the chain continues exactly from it; a full host base reseeds it."""
    rng = np.random.default_rng(34)
    ds = make_set(ctx, [300000, 5, 65536 * 2, 9999], seed=10, offsets=[0, 1, 0, 4])
    F = ctx.checkpoint(DEV, epoch=0)
    Fo = O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)
    _mutate(ds, _random_changes(ds, rng, 4))
    D1 = ctx.checkpoint_incremental(DEV, F, epoch=1)  # seeds the shadow from F's payload
    D1o = _odelta(ds, Fo, Fo, 1, checl.DIRTY_BYTES)
    _eq(D1.view(), D1o, "D1")
    full1 = O.checkpoint(oracle_entries(ds), device=DEV, epoch=1)
    _mutate(ds, _random_changes(ds, rng, 4))
    D2 = ctx.checkpoint_incremental(DEV, D1, epoch=2)  # shadow == D1's state
    D2o = _odelta(ds, D1o, full1, 2, checl.DIRTY_BYTES)
    _eq(D2.view(), D2o, "D2")
    full2 = O.checkpoint(oracle_entries(ds), device=DEV, epoch=2)
    # an older delta base: its state is not on the device -> the full image
    _mutate(ds, _random_changes(ds, rng, 2))
    X = ctx.checkpoint_incremental(DEV, D1, epoch=3)
    _eq(X.view(), O.checkpoint(oracle_entries(ds), device=DEV, epoch=3), "full fallback")
    assert X.header()["flags"] == 0
    full3 = O.checkpoint(oracle_entries(ds), device=DEV, epoch=3)
    _mutate(ds, _random_changes(ds, rng, 3))
    D4 = ctx.checkpoint_incremental(DEV, X, epoch=4)  # the fallback seeded the shadow
    _eq(D4.view(), _odelta(ds, full3, full3, 4, checl.DIRTY_BYTES), "D4")
    # back to the first full base: reseeded from its payload
    D5 = ctx.checkpoint_incremental(DEV, F, epoch=5)
    _eq(D5.view(), _odelta(ds, Fo, Fo, 5, checl.DIRTY_BYTES), "D5 on F")
    del full2
    release_all(ctx, ds)


def test_trim_releases_the_shadow(ctx):
    """checl_trim frees the exact rule's device copy of the last delta's state: a delta
    on that delta's base then has no state to compare with and is the full image; one on
    a full host base reseeds the copy and is exact again (reading 25)."""
    rng = np.random.default_rng(35)
    ds = make_set(ctx, [200000, 70001, 5], seed=12)
    F = ctx.checkpoint(DEV, epoch=0)
    Fo = O.checkpoint(oracle_entries(ds), device=DEV, epoch=0)
    _mutate(ds, _random_changes(ds, rng, 3))
    D1 = ctx.checkpoint_incremental(DEV, F, epoch=1)
    _eq(D1.view(), _odelta(ds, Fo, Fo, 1, checl.DIRTY_BYTES), "D1")
    ctx.trim()
    _mutate(ds, _random_changes(ds, rng, 3))
    X = ctx.checkpoint_incremental(DEV, D1, epoch=2)
    assert X.header()["flags"] == 0
    _eq(X.view(), O.checkpoint(oracle_entries(ds), device=DEV, epoch=2), "full after trim")
    ctx.trim()
    D3 = ctx.checkpoint_incremental(DEV, F, epoch=3)  # full host base: reseeded from F
    _eq(D3.view(), _odelta(ds, Fo, Fo, 3, checl.DIRTY_BYTES), "D3 on F")
    release_all(ctx, ds)
