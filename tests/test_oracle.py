"""Pins for the CPU oracle (-m "not gpu").

The oracle is checked against things other than itself (SURVEY.md §8(c) "What pins
each part"): published CRC32C vectors (north_star check value, RFC 3720 App. B.4),
two independent CRC32C implementations (the SSE4.2 crc32 instruction and GF(2)
polynomial division with Python integers), hand-derived layouts
(tests/golden/layout_cases.txt), and invariants — round trip, linearity, exhaustive
single-bit corruption localisation.
"""
import itertools
import os
import struct

import numpy as np
import pytest

from oracle import oracle as O
from tests.helpers import hwcrc

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _recipe(r: str) -> bytes:
    kind, *args = r.split(":")
    if kind == "ascii":
        return args[0].encode()
    if kind == "fill":
        return bytes([int(args[1], 16)]) * int(args[0])
    if kind == "range":
        return bytes(range(int(args[0]), int(args[1])))
    if kind == "rrange":
        return bytes(reversed(range(0, int(args[0]) + 1)))[: int(args[1])]
    raise ValueError(r)


def _vectors():
    out = []
    for line in open(os.path.join(GOLDEN, "crc32c_vectors.txt")):
        if line.startswith("#") or not line.strip():
            continue
        name, recipe, exp = (x.strip() for x in line.split("|"))
        out.append((name, _recipe(recipe), int(exp, 16)))
    return out


@pytest.mark.parametrize("name,data,expected", _vectors())
def test_crc32c_known_answers(name, data, expected):
    assert O.crc32c(data) == expected
    assert O.crc32c_bitwise(data) == expected
    assert hwcrc.poly_crc32c(data) == expected  # the independent pin itself agrees
    if hwcrc.available():
        assert hwcrc.hw_crc32c(data) == expected


def test_crc32c_tiny_brute_force_vs_polynomial_division():
    # every message of length 0..2 over all byte values, and random short ones
    msgs = [b""] + [bytes([a]) for a in range(256)]
    msgs += [bytes([a, b]) for a in range(0, 256, 7) for b in range(0, 256, 11)]
    rng = np.random.default_rng(7)
    msgs += [rng.integers(0, 256, int(n), dtype=np.uint8).tobytes() for n in rng.integers(3, 80, 200)]
    for m in msgs:
        p = hwcrc.poly_crc32c(m)
        assert O.crc32c(m) == p, m
        assert O.crc32c_bitwise(m) == p, m


@pytest.mark.skipif(not hwcrc.available(), reason="needs x86 SSE4.2")
def test_crc32c_vs_hardware_instruction_random_lengths():
    rng = np.random.default_rng(11)
    for n in list(range(0, 70)) + [255, 256, 257, 4095, 4096, 65535, 65536, 65537, 200003]:
        d = rng.integers(0, 256, n, dtype=np.uint8)
        assert O.crc32c(d) == hwcrc.hw_crc32c(d), n
    # SURVEY §8(c) cross-checked values
    assert O.crc32c(np.zeros(65536, np.uint8)) == 0x72C0C4A4
    assert O.crc32c(np.full(65536, 0xFF, np.uint8)) == 0x545A7F44
    assert O.crc32c((np.arange(65536) & 0xFF).astype(np.uint8)) == 0xA224AF3D
    assert O.crc32c(b"\x00") == 0x527D5351


def test_crc32c_linearity_invariant():
    # GF(2) linearity: crc(a ^ b) = crc(a) ^ crc(b) ^ crc(0^n) for equal lengths
    rng = np.random.default_rng(3)
    for n in (1, 4, 17, 1000, 65536):
        a = rng.integers(0, 256, n, dtype=np.uint8)
        b = rng.integers(0, 256, n, dtype=np.uint8)
        assert O.crc32c(a ^ b) == O.crc32c(a) ^ O.crc32c(b) ^ O.crc32c(np.zeros(n, np.uint8))


def _layout_cases():
    out = []
    for line in open(os.path.join(GOLDEN, "layout_cases.txt")):
        if line.startswith("#") or not line.strip():
            continue
        name, reg, offs, firsts, tail = (x.strip() for x in line.split("|"))
        regs = [tuple(int(v) for v in kv.split(":")) for kv in reg.split(",")] if reg else []
        offs = [int(v) for v in offs.split(",")] if offs else []
        firsts = [int(v) for v in firsts.split(",")] if firsts else []
        nch, crc_off, poff, pbytes, ibytes = (int(v) for v in tail.split())
        out.append((name, regs, offs, firsts, nch, crc_off, poff, pbytes, ibytes))
    return out


def _manifest(img):
    n = struct.unpack_from("<Q", img, 24)[0]
    recs = [struct.unpack_from("<QQQQIiQ", img, 128 + 48 * i) for i in range(n)]
    return recs


@pytest.mark.parametrize("case", _layout_cases(), ids=lambda c: c[0])
def test_layout_hand_derived(case):
    name, regs, offs, firsts, nch, crc_off, poff, pbytes, ibytes = case
    L = O.layout(regs)
    assert (L["n_chunks"], L["crc_off"], L["payload_off"], L["payload_bytes"], L["image_bytes"]) == (
        nch, crc_off, poff, pbytes, ibytes)
    if ibytes < (1 << 26):
        ents = [O.Entry(h, np.full(s, h & 0xFF, np.uint8)) for h, s in regs]
        img = O.checkpoint(ents, device=0, epoch=9).tobytes()
        assert len(img) == ibytes
        recs = _manifest(img)
        assert [r[0] for r in recs] == sorted(h for h, _ in regs)
        assert [r[2] for r in recs] == offs
        assert [r[3] for r in recs] == firsts


def test_layout_many_small_buffers_hand_derived():
    # 100 buffers of 1 B: offsets 256*i; crc_off = 128 + 4800 = 4928;
    # crc_end = 4928 + 400 = 5328 -> payload_off 8192; payload = 99*256 + 1.
    L = O.layout([(i + 1, 1) for i in range(100)])
    assert L == dict(n_buffers=100, n_chunks=100, crc_off=4928, payload_off=8192,
                     payload_bytes=25345, image_bytes=33537)


SIZES = [0, 1, 2, 15, 16, 17, 255, 256, 257, 65535, 65536, 65537]


def _check_image_by_definition(img: np.ndarray, ents, device, epoch):
    """Independent reading of FORMAT.md: header fields, each buffer's bytes at its
    offset, zero gaps, CRC table entries equal to the hardware CRC of each slice."""
    b = img.tobytes()
    assert b[:8] == b"CHECLIM1"
    ver, hb, cb, pa, n, nch, moff, crc_off, poff, pbytes, ibytes, dev, flags, ep = struct.unpack_from(
        "<IIIIQQQQQQQiIQ", b, 8)
    assert (ver, hb, cb, pa, moff, flags) == (1, 128, 65536, 256, 128, 0)
    assert (n, dev, ep, ibytes) == (len(ents), device, epoch, len(b))
    assert b[96:124] == bytes(28)
    srt = sorted(ents, key=lambda e: e.handle)
    recs = _manifest(b)
    covered = np.zeros(pbytes, dtype=bool)
    crcs = np.frombuffer(b, dtype="<u4", count=nch, offset=crc_off)
    for e, r in zip(srt, recs):
        h, size, off, first, fl, rdev, res = r
        assert (h, size, fl, rdev, res) == (e.handle, e.data.size, e.flags, device, 0)
        assert off % 256 == 0
        assert np.array_equal(img[poff + off: poff + off + size], e.data)
        covered[off: off + size] = True
        k = (size + 65535) // 65536
        offs = [poff + off + 65536 * j for j in range(k)]
        lens = [min(65536, size - 65536 * j) for j in range(k)]
        if k:
            if hwcrc.available():
                assert np.array_equal(crcs[first: first + k], hwcrc.hw_crc32c_many(img, offs, lens))
            else:
                assert [int(c) for c in crcs[first: first + k]] == [hwcrc.poly_crc32c(b[o:o + l]) for o, l in zip(offs, lens)]
    assert not img[poff: poff + pbytes][~covered].any(), "gap bytes must be zero"
    assert not img[crc_off + 4 * nch: poff].any()
    if hwcrc.available():
        meta = hwcrc.hw_crc32c(np.concatenate([img[:124], img[128:poff]]))
        assert struct.unpack_from("<I", b, 124)[0] == meta


def test_brute_force_registries_up_to_three_buffers():
    rng = np.random.default_rng(5)
    combos = [c for k in range(0, 4) for c in itertools.product(SIZES, repeat=k)]
    # all 1- and 2-buffer registries, and a deterministic third of the 3-buffer ones
    combos = [c for i, c in enumerate(combos) if len(c) < 3 or i % 3 == 0]
    for c in combos:
        handles = sorted(rng.choice(np.arange(1, 1000), size=len(c), replace=False).tolist(), reverse=True)
        ents = [O.Entry(int(h), rng.integers(0, 256, s, dtype=np.uint8), int(rng.integers(0, 2**32))) for h, s in zip(handles, c)]
        img = O.checkpoint(ents, device=3, epoch=len(c))
        _check_image_by_definition(img, ents, 3, len(c))
        st, rep, back = O.restore(img)
        assert st == 0 and rep["n_bad_chunks"] == 0
        srt = sorted(ents, key=lambda e: e.handle)
        assert [(e.handle, e.flags) for e in back] == [(e.handle, e.flags) for e in srt]
        for a, b in zip(back, srt):
            assert np.array_equal(a.data, b.data)


def test_round_trip_float_payloads_bit_exact():
    f = np.array([np.nan, -0.0, 0.0, np.inf, -np.inf, 1e-45, -1.5], dtype=np.float32)
    nan_payload = np.array([0x7FC00001, 0xFFFFFFFF, 0x7F800001], dtype=np.uint32).view(np.float32)
    ents = [O.Entry(1, f.view(np.uint8)), O.Entry(2, nan_payload.view(np.uint8)),
            O.Entry(3, np.random.default_rng(0).standard_normal(70001).astype(np.float64).view(np.uint8))]
    st, rep, back = O.restore(O.checkpoint(ents))
    assert st == 0
    for a, b in zip(back, ents):
        assert a.data.tobytes() == b.data.tobytes()


def _owner_chunk(img: bytes, pos: int):
    """(global chunk index, handle) owning payload byte pos, by FORMAT.md."""
    n = struct.unpack_from("<Q", img, 24)[0]
    poff, pbytes = struct.unpack_from("<QQ", img, 56)
    recs = _manifest(img)
    rel = pos - poff
    for i, (h, size, off, first, *_r) in enumerate(recs):
        end_pad = recs[i + 1][2] if i + 1 < n else pbytes
        if off <= rel < off + size:
            return first + (rel - off) // 65536, h
        if off + size <= rel < end_pad:
            return first + (size + 65535) // 65536 - 1, h
    raise AssertionError("byte outside payload")


def test_exhaustive_single_bit_flips_tiny_image():
    rng = np.random.default_rng(1)
    ents = [O.Entry(9, rng.integers(0, 256, 5, dtype=np.uint8)), O.Entry(2, np.zeros(0, np.uint8)),
            O.Entry(4, rng.integers(0, 256, 300, dtype=np.uint8))]
    img = O.checkpoint(ents, device=1, epoch=77)
    b = img.tobytes()
    poff = struct.unpack_from("<Q", b, 56)[0]
    assert len(b) > poff
    for pos in range(len(b)):
        for bit in range(8):
            bad = img.copy()
            bad[pos] ^= 1 << bit
            st, rep = O.validate(bad)
            if pos < poff:
                assert st == O.BAD_IMAGE, (pos, bit)
                continue
            assert st == 0
            st, rep, back = O.restore(bad)
            chunk, h = _owner_chunk(b, pos)
            assert st == O.CRC_MISMATCH and back == []
            assert (rep["n_bad_chunks"], rep["first_bad_chunk"], rep["first_bad_handle"]) == (1, chunk, h)


def test_multi_chunk_corruption_reports_lowest_chunk_and_count():
    rng = np.random.default_rng(2)
    ents = [O.Entry(1, rng.integers(0, 256, 200000, dtype=np.uint8)), O.Entry(2, rng.integers(0, 256, 70000, dtype=np.uint8))]
    img = O.checkpoint(ents)
    b = img.tobytes()
    poff = struct.unpack_from("<Q", b, 56)[0]
    bad = img.copy()
    # chunk 2 of handle 1 (global 2) and chunk 1 of handle 2 (global 5)
    bad[poff + 2 * 65536 + 7] ^= 0x40
    off2 = _manifest(b)[1][2]
    bad[poff + off2 + 65536 + 3] ^= 0x01
    st, rep, _ = O.restore(bad)
    assert st == O.CRC_MISMATCH
    assert (rep["n_bad_chunks"], rep["first_bad_chunk"], rep["first_bad_handle"]) == (2, 2, 1)


def test_bad_images_rejected():
    img = O.checkpoint([O.Entry(1, np.arange(10, dtype=np.uint8))])
    assert O.validate(img[:100])[0] == O.BAD_IMAGE
    assert O.validate(img[:-1])[0] == O.BAD_IMAGE
    assert O.validate(np.zeros(4096, np.uint8))[0] == O.BAD_IMAGE
    ok = O.validate(np.concatenate([img, np.zeros(7, np.uint8)]))[0]
    assert ok == 0  # a longer buffer is accepted; image_bytes bounds the image


def test_invalid_registries_rejected():
    with pytest.raises(ValueError):
        O.checkpoint([O.Entry(0, np.zeros(3, np.uint8))])
    with pytest.raises(ValueError):
        O.checkpoint([O.Entry(4, np.zeros(3, np.uint8)), O.Entry(4, np.zeros(1, np.uint8))])


def test_synth_slices_match_whole_buffer():
    import synth
    full = synth.fill_bytes(70001, 9, 4)
    for off, n in [(0, 1), (7, 33), (8, 8), (12345, 999), (69990, 11)]:
        assert np.array_equal(synth.fill_slice(off, n, 9, 4), full[off:off + n])
