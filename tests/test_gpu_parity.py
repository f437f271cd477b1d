"""-m gpu: the CUDA path (through the C ABI) against the CPU oracle, bit-exact.

Checkpoint images (header, manifest, CRC table, payload) must equal the oracle's
image byte for byte; restore must reproduce every buffer and report exactly the
oracle's first bad chunk / handle / count on corrupted images. Sizes span several
stripes, chunks and staging slots, with ragged tails, zero-size buffers and
misaligned views.
"""
import itertools
import struct

import numpy as np
import pytest

import synth
from oracle import oracle as O
from tests.gpu_util import bound_bytes, make_set, oracle_entries, release_all

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

DEV = 0
SIZES = [0, 1, 2, 15, 16, 17, 255, 256, 257, 65535, 65536, 65537]


@pytest.fixture()
def ctx():
    c = checl.Context()
    yield c
    c.close()


def _ckpt_equal(ctx, ds, epoch=5):
    img = ctx.checkpoint(DEV, epoch=epoch)
    want = O.checkpoint(oracle_entries(ds), device=DEV, epoch=epoch)
    got = img.view()
    assert got.size == want.size
    if not np.array_equal(got, want):
        bad = np.nonzero(got != want)[0]
        raise AssertionError(f"image differs at {bad.size} bytes, first {bad[:8]}")
    return img, want


def test_device_fill_matches_synth_generator():
    for kind in (checl.FILL_RANDOM, checl.FILL_FLOAT, checl.FILL_ZEROS):
        for n in (1, 7, 8, 9, 4097, 1 << 20):
            for off in (0, 1, 4):
                b = torch.empty(n + off + 8, dtype=torch.uint8, device=DEV)
                v = b[off:off + n]
                checl.debug_fill(v, 11, 3, kind)
                want = synth.fill_bytes(n, 11, 3, ["random", "float", "zeros"][kind])
                assert np.array_equal(v.cpu().numpy(), want), (kind, n, off)


def test_edge_size_registries_bit_exact(ctx):
    combos = [c for k in (1, 2, 3) for c in itertools.product(SIZES, repeat=k)]
    combos = [c for i, c in enumerate(combos) if len(c) < 3 or i % 7 == 0]
    for i, c in enumerate(combos):
        ds = make_set(ctx, c, seed=i, offsets=[(i + j) % 3 * 4 + (j % 2) for j in range(len(c))])
        img, _ = _ckpt_equal(ctx, ds, epoch=i)
        img.free()
        release_all(ctx, ds)


def test_empty_registry_bit_exact(ctx):
    img = ctx.checkpoint(DEV, epoch=1)
    assert np.array_equal(img.view(), O.checkpoint([], device=DEV, epoch=1))
    rep = ctx.restore(img, DEV)
    assert rep.n_buffers == 0


RAGGED = [65536 * 5 + 1, 2048 * 7 + 3, 2047, 2049, 131072, 4096 + 12, 65536 * 3 - 1, 100000, 3, 0, 65536 + 2048 + 5]


@pytest.mark.parametrize("misalign", [0, 1, 4, 8])
def test_multi_tile_ragged_bit_exact(ctx, misalign):
    ds = make_set(ctx, RAGGED, seed=42, offsets=[misalign] * len(RAGGED))
    img, _ = _ckpt_equal(ctx, ds)
    img.free()


@pytest.mark.parametrize("kind", [checl.FILL_FLOAT, checl.FILL_ZEROS])
def test_data_kinds_bit_exact(ctx, kind):
    ds = make_set(ctx, RAGGED, seed=9, kind=kind)
    img, _ = _ckpt_equal(ctx, ds)
    img.free()


def test_special_float_payloads_round_trip(ctx):
    f = torch.tensor([float("nan"), -0.0, 0.0, float("inf"), -float("inf"), 1e-45, -1.5] * 1000,
                     dtype=torch.float32, device=DEV)
    raw = torch.tensor([0x7FC00001, -1, 0x7F800001] * 999, dtype=torch.int32, device=DEV)
    h1, h2 = ctx.register(f), ctx.register(raw)
    want = [f.view(torch.uint8).cpu().numpy(), raw.view(torch.uint8).cpu().numpy()]
    img = ctx.checkpoint(DEV)
    assert np.array_equal(img.view(), O.checkpoint([O.Entry(h1, want[0]), O.Entry(h2, want[1])], device=DEV))
    ctx.restore(img, DEV)
    assert np.array_equal(bound_bytes(ctx, h1), want[0]) and np.array_equal(bound_bytes(ctx, h2), want[1])


@pytest.mark.parametrize("slot,n", [(131072, 1), (131072, 2), (196608, 3), (1 << 20, 2)])
def test_small_staging_slots_bit_exact_and_restore(ctx, slot, n):
    ctx.set_staging(slot, n)
    ds = make_set(ctx, RAGGED + [700001, 65536 * 4], seed=5, offsets=[1] * 13)
    img, want = _ckpt_equal(ctx, ds)
    old = [ctx.translate(h)[0] for h in ds.handles]
    rep = ctx.restore(img, DEV)
    assert rep.n_bad_chunks == 0 and rep.n_buffers == len(ds.handles)
    for h, b, o in zip(ds.handles, ds.host, old):
        ptr, nb, d = ctx.translate(h)
        assert nb == b.size and d == DEV
        assert (ptr == 0) if nb == 0 else (ptr != o)
        assert np.array_equal(bound_bytes(ctx, h), b)
    img.free()


def test_device_image_equals_host_image(ctx):
    ds = make_set(ctx, RAGGED, seed=3, offsets=[4] * len(RAGGED))
    himg, want = _ckpt_equal(ctx, ds, epoch=77)
    dimg = ctx.checkpoint_device(DEV, epoch=77)
    info = dimg.info()
    assert info["location"] == checl.IMAGE_DEVICE and info["image_bytes"] == want.size
    h2 = dimg.to_host()
    assert np.array_equal(h2.view(), want)
    rep = ctx.restore(dimg, DEV)
    assert rep.n_bad_chunks == 0
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)


def test_restore_oracle_image_into_fresh_context():
    rng = np.random.default_rng(4)
    ents = [O.Entry(h, rng.integers(0, 256, s, dtype=np.uint8), h * 3) for h, s in
            [(3, 70000), (8, 0), (11, 5), (40, 65536 * 2 + 17)]]
    img_bytes = O.checkpoint(ents, device=DEV, epoch=12)
    with checl.Context() as c2:
        img = checl.Image.wrap(img_bytes)
        rep = c2.restore(img, DEV)
        assert rep.n_buffers == 4 and rep.n_bad_chunks == 0
        for e in ents:
            ptr, nb, d = c2.translate(e.handle)
            assert nb == e.data.size
            assert np.array_equal(bound_bytes(c2, e.handle), e.data)
        # ids never reused: a new registration gets an id above the image's maximum
        t = torch.zeros(4, dtype=torch.uint8, device=DEV)
        assert c2.register(t) == 41
        img.free()


def _payload_positions(img: np.ndarray, rng, n):
    poff, pbytes = struct.unpack_from("<QQ", img.tobytes()[:128], 56)
    return [int(poff + x) for x in rng.integers(0, pbytes, n)]


def test_corruption_reports_match_oracle_and_nothing_rebound(ctx):
    ds = make_set(ctx, RAGGED, seed=8)
    img, want = _ckpt_equal(ctx, ds)
    before = {h: ctx.translate(h) for h in ds.handles}
    rng = np.random.default_rng(0)
    for trial in range(40):
        nflip = 1 + trial % 4
        pos = _payload_positions(want, rng, nflip)
        bad = want.copy()
        for p in pos:
            bad[p] ^= np.uint8(1 << int(rng.integers(0, 8)))
        st, orep, _ = O.restore(bad)
        wimg = checl.Image.wrap(bad)
        if st == 0:
            ctx.restore(wimg, DEV)  # flips cancelled out (same byte twice): must succeed
            before = {h: ctx.translate(h) for h in ds.handles}
            continue
        assert st == O.CRC_MISMATCH
        with pytest.raises(checl.CheclError) as ei:
            ctx.restore(wimg, DEV)
        e = ei.value
        assert e.status == checl.ERR_CRC_MISMATCH
        r = e.report
        assert (r.n_bad_chunks, r.first_bad_chunk, r.first_bad_handle) == (
            orep["n_bad_chunks"], orep["first_bad_chunk"], orep["first_bad_handle"])
        assert {h: ctx.translate(h) for h in ds.handles} == before, "nothing may be rebound"
        wimg.free()


def test_exhaustive_single_bit_flips_tiny_image(ctx):
    ds = make_set(ctx, [5, 0, 300], seed=1)
    img, want = _ckpt_equal(ctx, ds, epoch=2)
    poff = struct.unpack_from("<Q", want.tobytes(), 56)[0]
    before = {h: ctx.translate(h) for h in ds.handles}
    for pos in range(want.size):
        bits = range(8) if pos >= poff or pos < 512 else (pos % 8,)  # header, manifest, CRC table: every bit; zero pad: one bit
        for bit in bits:
            bad = want.copy()
            bad[pos] ^= np.uint8(1 << bit)
            st, orep, _ = O.restore(bad)
            wimg = checl.Image.wrap(bad)
            with pytest.raises(checl.CheclError) as ei:
                ctx.restore(wimg, DEV)
            wimg.free()
            if pos < poff:
                assert st == O.BAD_IMAGE and ei.value.status == checl.ERR_BAD_IMAGE, (pos, bit)
            else:
                r = ei.value.report
                assert ei.value.status == checl.ERR_CRC_MISMATCH
                assert (r.n_bad_chunks, r.first_bad_chunk, r.first_bad_handle) == (
                    orep["n_bad_chunks"], orep["first_bad_chunk"], orep["first_bad_handle"]), (pos, bit)
    assert {h: ctx.translate(h) for h in ds.handles} == before


def test_device_image_corruption_detected(ctx):
    ds = make_set(ctx, [200000, 70000], seed=2)
    dimg = ctx.checkpoint_device(DEV)
    host = dimg.to_host().view().copy()
    poff = struct.unpack_from("<Q", host.tobytes(), 56)[0]
    dimg.corrupt(poff + 65536 * 2 + 9, 0x10)  # chunk 2 of the first buffer
    with pytest.raises(checl.CheclError) as ei:
        ctx.restore(dimg, DEV)
    r = ei.value.report
    assert (r.n_bad_chunks, r.first_bad_chunk, r.first_bad_handle) == (1, 2, ds.handles[0])


def test_migrate_same_device_moves_to_new_buffers(ctx):
    ds = make_set(ctx, RAGGED, seed=6, offsets=[1] * len(RAGGED))
    old = {h: ctx.translate(h) for h in ds.handles}
    rep = ctx.migrate(DEV, DEV)
    assert rep.n_bad_chunks == 0 and rep.n_buffers == len(RAGGED)
    for h, b in zip(ds.handles, ds.host):
        ptr, nb, d = ctx.translate(h)
        assert nb == b.size and d == DEV
        if nb:
            assert ptr != old[h][0]
        assert np.array_equal(bound_bytes(ctx, h), b)
    # second migration frees the library-owned buffers of the first
    rep = ctx.migrate(DEV, DEV)
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)


def test_restore_twice_and_release_owned(ctx):
    ds = make_set(ctx, [1 << 20, 12345], seed=10)
    img = ctx.checkpoint(DEV)
    ctx.restore(img, DEV)
    ctx.restore(img, DEV)
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)
    for h in ds.handles:
        ctx.release(h)
    with pytest.raises(checl.CheclError):
        ctx.translate(ds.handles[0])


def test_restart_loop_release_all_then_restore(ctx):
    """bench.py restart mode (L16 restart steps 2-3): checkpoint -> release every
    handle -> restore re-creates them, repeated on one device image. Every image equals
    the oracle's (same ids, flags, bytes) and the re-created buffers hold the bytes."""
    ds = make_set(ctx, RAGGED, seed=21, offsets=[3] * len(RAGGED))
    want = O.checkpoint(oracle_entries(ds), device=DEV, epoch=1)
    img = ctx.checkpoint_device(DEV, epoch=1)
    assert np.array_equal(img.to_host().view(), want)
    for h in ds.handles:
        ctx.release(h)
    del ds.tensors[:], ds.bases[:]  # the application's buffers are gone
    for epoch in (2, 3, 4):
        rep = ctx.restore(img, DEV)
        assert rep.n_bad_chunks == 0 and rep.n_buffers == len(RAGGED)
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b)
        ctx.checkpoint(DEV, epoch=epoch, into=img)
        assert np.array_equal(img.to_host().view(), O.checkpoint(oracle_entries(ds), device=DEV, epoch=epoch))
        for h in ds.handles:
            ctx.release(h)
    assert ctx.count(DEV)[0] == 0


def test_stats_accumulate_deferred_event_spans(ctx):
    """Event spans are read lazily (next call / query): per-call timings and the
    cumulative checl_stats agree, with or without a query after every call."""
    make_set(ctx, [1 << 22, 12345, 0], seed=31)
    img = ctx.checkpoint_device(DEV, epoch=1)
    ctx.reset_stats()
    ks, rs = [], []
    for e in range(3):
        ctx.checkpoint(DEV, epoch=e, into=img)
        ks.append(ctx.last_timing())
        ctx.restore(img, DEV)
        rs.append(ctx.last_timing())
    s0, s1 = ctx.stats(checl.STATS_CHECKPOINT), ctx.stats(checl.STATS_RESTORE)
    assert s0["n_calls"] == 3 and s1["n_calls"] == 3
    assert all(t["kernel_ms"] > 0 and t["n_kernels"] >= 1 for t in ks + rs)
    assert s0["kernel_ms"] == pytest.approx(sum(t["kernel_ms"] for t in ks), rel=1e-12)
    assert s1["kernel_ms"] == pytest.approx(sum(t["kernel_ms"] for t in rs), rel=1e-12)
    assert s0["n_kernels"] == sum(t["n_kernels"] for t in ks)
    ctx.reset_stats()
    for e in range(4):  # no query in between: each call reads the previous call's spans
        ctx.checkpoint(DEV, epoch=e, into=img)
        ctx.restore(img, DEV)
    last = ctx.last_timing()
    s0, s1 = ctx.stats(checl.STATS_CHECKPOINT), ctx.stats(checl.STATS_RESTORE)
    assert s0["n_calls"] == 4 and s1["n_calls"] == 4 and last["kernel_ms"] > 0
    assert s0["kernel_ms"] > 0 and s1["kernel_ms"] >= last["kernel_ms"]
    assert ctx.stats(checl.STATS_INCREMENTAL)["n_calls"] == 0
    with pytest.raises(checl.CheclError):
        ctx.stats(4)


def test_checkpoint_into_reuses_and_grows(ctx):
    ds = make_set(ctx, [1000, 70000], seed=12)
    img = ctx.checkpoint(DEV, epoch=1)
    ds2 = make_set(ctx, [65536 * 9 + 7], seed=13)
    ctx.checkpoint(DEV, epoch=2, into=img)
    allset = oracle_entries(ds) + oracle_entries(ds2)
    assert np.array_equal(img.view(), O.checkpoint(allset, device=DEV, epoch=2))


def test_c1_vectoradd_round_trip(ctx):
    w = synth.c1_vectoradd()
    ds = make_set(ctx, [b.size for b in w.buffers], seed=w.seed, kind=checl.FILL_FLOAT)
    img, _ = _ckpt_equal(ctx, ds)
    ctx.restore(img, DEV)
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)


def test_c2_sdk_mix_full_size_bit_exact(ctx):
    """configs[1] at full size: the pinned host image and the HBM image (the bench's
    `value` path: tma_kernel into device memory) both equal the oracle's image byte for
    byte."""
    w = synth.c2_sdk_mix()
    ds = make_set(ctx, [b.size for b in w.buffers], seed=w.seed)
    img, want = _ckpt_equal(ctx, ds)
    dimg = ctx.checkpoint_device(DEV, epoch=5)
    h = dimg.to_host()
    assert np.array_equal(h.view(), want), "HBM image != oracle image"
    h.free()
    rep = ctx.restore(dimg, DEV)
    assert rep.n_bad_chunks == 0 and rep.n_chunks == 7070
    for h, t in zip(ds.handles, ds.tensors):
        ptr, nb, _ = ctx.translate(h)
        assert checl.debug_compare(DEV, ptr, t.data_ptr(), nb) == 0
    rep = ctx.restore(img, DEV)
    for h, t in zip(ds.handles, ds.tensors):
        ptr, nb, _ = ctx.translate(h)
        assert checl.debug_compare(DEV, ptr, t.data_ptr(), nb) == 0


def _parallel(fn, items, threads=8):
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(threads) as ex:
        return list(ex.map(fn, items))


def test_c3_handle_stress_full_size(ctx):
    """configs[2] at full size (10,000 odd buffers, 5.35 GB), every byte: layout and
    manifest from the oracle; every buffer's payload equals the synth generator's bytes
    (synth.fill_bytes); every one of the 86,582 CRC-table entries equals the x86 SSE4.2
    crc32 instruction's CRC32C of its chunk (tests/helpers, an implementation
    independent of the oracle and the product); the oracle's CRC on 300 sampled
    buffers; the HBM image (the bench's launch configuration) equals the host image
    byte for byte; round trip on all."""
    from tests.helpers import hwcrc
    if not hwcrc.available():
        pytest.skip("needs the SSE4.2 crc32 instruction")
    w = synth.c3_handle_stress()
    sizes = [b.size for b in w.buffers]
    big = torch.empty(sum(s + 256 for s in sizes), dtype=torch.uint8, device=DEV)
    handles, views, pos = [], [], 0
    for i, s in enumerate(sizes):
        off = pos + (i % 5)  # varied alignment
        v = big[off:off + s]
        checl.debug_fill(v, w.seed, i)
        views.append(v)
        pos += s + 256
    torch.cuda.synchronize()
    handles = [ctx.register(v, 7) for v in views]
    img = ctx.checkpoint(DEV, epoch=3)
    got = img.view()
    L = O.layout(list(zip(handles, sizes)))
    assert got.size == L["image_bytes"]
    hdr = got[:128].tobytes()
    assert struct.unpack_from("<QQQQQQQ", hdr, 24) == (len(sizes), L["n_chunks"], 128, L["crc_off"],
                                                        L["payload_off"], L["payload_bytes"], L["image_bytes"])
    recs = [struct.unpack_from("<QQQQIiQ", got, 128 + 48 * i) for i in range(len(sizes))]
    crcs = np.frombuffer(got, dtype="<u4", count=L["n_chunks"], offset=L["crc_off"])
    def buffer_ok(i):
        h, size, off, first, fl, dv, _ = recs[i]
        p0 = L["payload_off"] + off
        return (h, size, fl, dv) == (handles[i], sizes[i], 7, DEV) and np.array_equal(
            got[p0:p0 + size], synth.fill_bytes(size, w.seed, i))
    bad = [i for i, ok in zip(range(len(sizes)), _parallel(buffer_ok, range(len(sizes)))) if not ok]
    assert not bad, bad[:10]
    offs, lens = [], []
    for h, size, off, first, fl, dv, _ in recs:
        for k in range((size + 65535) // 65536):
            offs.append(L["payload_off"] + off + 65536 * k)
            lens.append(min(65536, size - 65536 * k))
    assert len(offs) == L["n_chunks"]
    hw = hwcrc.hw_crc32c_many(got, offs, lens)
    assert np.array_equal(hw, crcs), int(np.count_nonzero(hw != crcs))
    rng = np.random.default_rng(1)
    for i in rng.choice(len(sizes), 300, replace=False):
        h, size, off, first, fl, dv, _ = recs[i]
        data = synth.fill_bytes(size, w.seed, int(i))
        for k in range((size + 65535) // 65536):
            assert int(crcs[first + k]) == O.crc32c(data[k * 65536:(k + 1) * 65536])
    dimg = ctx.checkpoint_device(DEV, epoch=3)
    hd = dimg.to_host()
    assert np.array_equal(hd.view(), got), "HBM image != host image"
    hd.free()
    dimg.free()
    # meta CRC vs the oracle's definition on the image's own bytes
    st, _ = O.validate(got)
    assert st == 0
    rep = ctx.restore(img, DEV)
    assert rep.n_bad_chunks == 0 and rep.n_buffers == len(sizes)
    nd = 0
    for h, v in zip(handles, views):
        ptr, nb, _ = ctx.translate(h)
        nd += checl.debug_compare(DEV, ptr, v.data_ptr(), nb)
    assert nd == 0


def test_repeated_device_restores_reuse_chunk_list_and_status(ctx):
    """The bench loop (checkpoint_into a device image -> restore, repeated): restores
    alternate between two allocations and skip the chunk-list expansion once the
    scratch list matches; the verify status is published by the last CTA and left at
    rest, also after a failing restore (DESIGN.md §5 "Restore launches")."""
    sizes = [1 << 20, 70001, 0, 3 * 65536 + 5, 4097]
    ds = make_set(ctx, sizes, seed=21, offsets=[0, 4, 0, 1, 0])
    dimg = ctx.checkpoint_device(DEV, epoch=1)
    kernels = []
    for i in range(6):
        ctx.checkpoint(DEV, epoch=i + 2, into=dimg)
        ctx.restore(dimg, DEV)
        kernels.append(ctx.last_timing()["n_kernels"])
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b), (i, h)
    assert kernels[-1] == 1 and kernels[-2] == 1, kernels  # verify only, no expansion
    host = dimg.to_host().view().copy()
    poff = struct.unpack_from("<Q", host.tobytes(), 56)[0]
    bad = poff + 65536 * 16 + 256 + 3  # second buffer (offset 1 MiB), chunk 0 -> global chunk 16
    for rep in range(2):
        dimg.corrupt(bad, 0x01)
        with pytest.raises(checl.CheclError) as ei:
            ctx.restore(dimg, DEV)
        r = ei.value.report
        assert (r.n_bad_chunks, r.first_bad_chunk, r.first_bad_handle) == (1, 16, ds.handles[1]), rep
        dimg.corrupt(bad, 0x01)  # undo: the next restore must not see stale status
        ctx.restore(dimg, DEV)
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b), (rep, h)
    # a host image and a device image alternating share the status words
    himg = ctx.checkpoint(DEV, epoch=9)
    for i in range(3):
        ctx.restore(himg if i % 2 else dimg, DEV)
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b), (i, h)


def test_same_header_other_manifest_takes_the_long_way(ctx):
    """Restore reuses the parse, segments and chunk list of the device's last restore
    when the image header matches (DESIGN.md §5 "Restore fast path"), comparing the
    manifest while K2 runs. Two oracle images with identical headers but different
    manifests (other handles, other flags): each restore must bind exactly its own
    image's handles, flags and bytes."""
    rng = np.random.default_rng(71)
    sizes = [70001, 3, 65536 * 2 + 9]
    data = [rng.integers(0, 256, s, dtype=np.uint8) for s in sizes]
    A = O.checkpoint([O.Entry(h, d, 5) for h, d in zip((11, 12, 13), data)], device=DEV, epoch=1)
    B = O.checkpoint([O.Entry(h, d ^ 0x5A, 5) for h, d in zip((21, 22, 23), data)], device=DEV, epoch=2)
    C = O.checkpoint([O.Entry(h, d, 6) for h, d in zip((11, 12, 13), data)], device=DEV, epoch=3)  # flags only
    assert A[:88].tobytes() == B[:88].tobytes() == C[:88].tobytes()
    for rnd in range(2):
        for img, hs, want, fl in ((A, (11, 12, 13), data, 5), (B, (21, 22, 23), [d ^ 0x5A for d in data], 5),
                                  (A, (11, 12, 13), data, 5), (C, (11, 12, 13), data, 6)):
            rep = ctx.restore(checl.Image.wrap(img), DEV)
            assert rep.n_bad_chunks == 0 and rep.n_buffers == 3
            for h, d in zip(hs, want):
                assert np.array_equal(bound_bytes(ctx, h), d), (rnd, h)
        # the image checkpointed now holds every live handle with its flags
        got = ctx.checkpoint(DEV, epoch=9).view()
        st, _, ents = O.restore(got)
        assert st == 0 and {e.handle: e.flags for e in ents} == {11: 6, 12: 6, 13: 6, 21: 5, 22: 5, 23: 5}


def test_restore_fast_paths_follow_registry_changes(ctx):
    """A checkpoint/restore loop takes the fast paths (cached layout, chunk-list key,
    in-place rebinding); a registration or release in between must send the next
    commit the long way, and every handle must stay exact."""
    sizes = [1 << 20, 70001, 0, 3 * 65536 + 5, 4097]
    ds = make_set(ctx, sizes, seed=72, offsets=[0, 4, 0, 1, 0])
    dimg = ctx.checkpoint_device(DEV, epoch=1)
    extra = []
    for i in range(8):
        ctx.checkpoint(DEV, epoch=i + 2, into=dimg)
        ctx.restore(dimg, DEV)
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b), (i, h)
        if i == 3:  # a new registration: the next image has another layout
            t = torch.full((777,), 9, dtype=torch.uint8, device=DEV)
            extra.append((ctx.register(t), t))
        if i == 5:  # and its release: back to the first layout
            h, t = extra.pop()
            ctx.release(h)
    n, total = ctx.count(DEV)
    assert n == len(sizes) and total == sum(sizes)
    release_all(ctx, ds)


def test_large_table_meta_crc_on_gpu(ctx):
    """A device image whose CRC table is at least 128 KB has its meta CRC computed on
    the GPU (meta_crc_kernel: per-thread slicing-by-4 pieces combined by CRC linearity,
    DESIGN.md §5 "Finalize"): 40 000 one-chunk buffers (a 160 KB table, odd sizes,
    misaligned views), host and HBM images equal the oracle's byte for byte."""
    rng = np.random.default_rng(81)
    n = 40000
    sizes = [int(x) for x in rng.integers(1, 200, n)]
    big = torch.empty(sum(sizes) + 8 * n, dtype=torch.uint8, device=DEV)
    views, pos = [], 0
    for i, s in enumerate(sizes):
        off = pos + (i % 7)
        views.append(big[off:off + s])
        pos += s + 8
    checl.debug_fill(big, 81, 0)
    torch.cuda.synchronize()
    handles = [ctx.register(v, i & 0xFF) for i, v in enumerate(views)]
    host = big.cpu().numpy()
    ents, pos = [], 0
    for i, (h, s) in enumerate(zip(handles, sizes)):
        off = pos + (i % 7)
        ents.append(O.Entry(h, host[off:off + s], i & 0xFF))
        pos += s + 8
    want = O.checkpoint(ents, device=DEV, epoch=17)
    dimg = ctx.checkpoint_device(DEV, epoch=17)
    h = dimg.to_host()
    assert np.array_equal(h.view(), want), "HBM image (GPU meta CRC) != oracle image"
    for e in (18, 19):  # repeated: the manifest is not rewritten, the epoch term changes
        ctx.checkpoint(DEV, epoch=e, into=dimg)
        h2 = dimg.to_host()
        assert np.array_equal(h2.view(), O.checkpoint(ents, device=DEV, epoch=e)), e
        h2.free()
    h.free()
    img = ctx.checkpoint(DEV, epoch=17)
    assert np.array_equal(img.view(), want)


@pytest.mark.parametrize("total_mib", [40, 150, 600])
def test_work_split_regimes_device_image_bit_exact(ctx, total_mib):
    """The TMA kernel's work split changes with the launch size (static
    stretches below 16 rounds per warp, 500 permille static + blocks of 4 below 64,
    + blocks of 8 below 256; C3-sized launches are covered by test_gpu_fullsize). One
    launch per regime over odd-sized buffers, some misaligned (register-path rounds
    beside bulk rounds, chunks split between static stretches and dynamic blocks): the
    device image equals the oracle's byte for byte and a restore reproduces every
    buffer."""
    rng = np.random.default_rng(total_mib)
    sizes, left = [], total_mib << 20
    while left > 0:
        s = int(min(left, rng.integers(1 << 18, 9 << 20))) | 1
        sizes.append(s)
        left -= s
    sizes[3:3] = [0, 5, 4096, 65537]
    offsets = [int(rng.choice([0, 0, 0, 1, 4, 8])) for _ in sizes]
    ds = make_set(ctx, sizes, seed=total_mib, offsets=offsets)
    want = O.checkpoint(oracle_entries(ds), device=DEV, epoch=7)
    img = ctx.checkpoint_device(DEV, epoch=7)
    got = img.to_host().view()
    assert got.size == want.size
    if not np.array_equal(got, want):
        bad = np.nonzero(got != want)[0]
        raise AssertionError(f"image differs at {bad.size} bytes, first {bad[:8]}")
    for t in ds.tensors:  # the application's bytes change; the restore brings them back
        t.zero_()
    rep = ctx.restore(img, DEV)
    assert rep.n_bad_chunks == 0 and rep.n_buffers == len(sizes)
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b)
    img.free()
    release_all(ctx, ds)
