"""Pins for the incremental-checkpoint oracle (PAPER.md L45
§IV-D "only the OpenCL objects updated since the last checkpoint"), -m "not gpu".
Two rules decide "updated" (FORMAT.md "Present set"): the CRC rule (DESIGN.md
reading 21) and the bytes rule (reading 25, the plain definition; pinned at the end
by byte differences computed here with numpy and by merge == full image even for a
change the CRC cannot see).

Checked against things other than the oracle's own incremental code: an
independent reading of FORMAT.md "Incremental images" (header fields, bitmap,
spans recomputed here from the manifest formulas, meta CRC and base-table CRC with
the SSE4.2 crc32 instruction), the closed forms of the two extreme cases (nothing
changed: empty payload; everything changed: the compacted payload *is* the full
payload), brute force over single-byte changes (exactly the owning chunk is
present), and the round trip merge(F, D) == the full image of the new state
(checkpoint itself is pinned in test_oracle.py).
"""
import itertools
import struct

import numpy as np
import pytest

from oracle import oracle as O
from tests.helpers import hwcrc

SIZES = [0, 1, 17, 256, 257, 65535, 65536, 65537, 131075]


def _crc(b: bytes) -> int:
    return hwcrc.hw_crc32c(np.frombuffer(b, np.uint8)) if hwcrc.available() else hwcrc.poly_crc32c(b)


def _align(x, a):
    return (x + a - 1) // a * a


def _spans(ents):
    """[(k, start, stop)] of every chunk, from FORMAT.md's formulas (handle order)."""
    srt = sorted(ents, key=lambda e: e.handle)
    offs, end = [], 0
    for i, e in enumerate(srt):
        off = 0 if i == 0 else _align(end, 256)
        offs.append(off)
        end = off + e.data.size
    full = end if srt else 0
    out, k = [], 0
    for i, e in enumerate(srt):
        nch = (e.data.size + 65535) // 65536
        for j in range(nch):
            start = offs[i] + 65536 * j
            stop = start + 65536 if j + 1 < nch else (offs[i + 1] if i + 1 < len(srt) else full)
            out.append((k, start, stop))
            k += 1
    return out


def _check_delta_by_definition(delta: np.ndarray, base: np.ndarray, new_full: np.ndarray, ents_now, present,
                               rule: int = 0):
    """Independent reading of FORMAT.md "Incremental images"."""
    d, f, b = delta.tobytes(), new_full.tobytes(), base.tobytes()
    nch, crc_off = struct.unpack_from("<QQ", f, 32)[0], struct.unpack_from("<Q", f, 48)[0]
    f_poff = struct.unpack_from("<Q", f, 56)[0]
    assert d[:56] == f[:56]  # magic .. crc_off identical to the full image's
    poff, pbytes, ibytes = struct.unpack_from("<QQQ", d, 56)
    assert d[80:84] == f[80:84] and d[88:96] == f[88:96]  # device, epoch
    flags, = struct.unpack_from("<I", d, 84)
    base_epoch, base_tab, res1, n_present, res2 = struct.unpack_from("<QIIQI", d, 96)
    assert (flags, res1, res2) == (1, rule, 0)  # res1 = dirty_rule
    assert base_epoch == struct.unpack_from("<Q", b, 88)[0]
    assert base_tab == _crc(b[crc_off: crc_off + 4 * nch])
    map_bytes = (nch + 7) // 8
    assert poff == _align(crc_off + 4 * nch + map_bytes, 4096)
    assert d[128:crc_off + 4 * nch] == f[128:crc_off + 4 * nch]  # manifest + CRC table of this epoch
    bits = np.unpackbits(np.frombuffer(d[crc_off + 4 * nch: crc_off + 4 * nch + map_bytes], np.uint8), bitorder="little")
    assert sorted(np.nonzero(bits)[0].tolist()) == sorted(present)
    assert n_present == len(present)
    assert d[crc_off + 4 * nch + map_bytes: poff] == bytes(poff - crc_off - 4 * nch - map_bytes)
    want = b"".join(f[f_poff + s: f_poff + t] for k, s, t in _spans(ents_now) if k in set(present))
    assert pbytes == len(want) and ibytes == poff + pbytes == len(d)
    assert d[poff:] == want
    assert struct.unpack_from("<I", d, 124)[0] == _crc(d[:124] + d[128:poff])


def _mutate(ents, changes):
    out = [O.Entry(e.handle, e.data.copy(), e.flags) for e in ents]
    for i, pos, x in changes:
        out[i].data[pos] ^= x
    return out


def test_unchanged_state_gives_empty_delta():
    rng = np.random.default_rng(21)
    for c in itertools.product(SIZES, repeat=2):
        ents = [O.Entry(7, rng.integers(0, 256, c[0], dtype=np.uint8), 5), O.Entry(3, rng.integers(0, 256, c[1], dtype=np.uint8))]
        F = O.checkpoint(ents, device=2, epoch=10)
        D = O.checkpoint_incremental(ents, F, device=2, epoch=11)
        _check_delta_by_definition(D, F, O.checkpoint(ents, device=2, epoch=11), ents, [])
        st, M = O.merge(F, D)
        assert st == 0 and np.array_equal(M, O.checkpoint(ents, device=2, epoch=11))


def test_everything_changed_delta_payload_is_the_full_payload():
    rng = np.random.default_rng(22)
    ents = [O.Entry(1, rng.integers(0, 256, 200003, dtype=np.uint8)), O.Entry(2, rng.integers(0, 256, 77, dtype=np.uint8)),
            O.Entry(4, np.zeros(0, np.uint8)), O.Entry(9, rng.integers(0, 256, 65536, dtype=np.uint8))]
    F = O.checkpoint(ents, epoch=1)
    now = [O.Entry(e.handle, ~e.data, e.flags) for e in ents]
    D = O.checkpoint_incremental(now, F, epoch=2)
    F2 = O.checkpoint(now, epoch=2)
    poff_f, pbytes_f = struct.unpack_from("<QQ", F2.tobytes(), 56)
    poff_d, pbytes_d = struct.unpack_from("<QQ", D.tobytes(), 56)
    nch = struct.unpack_from("<Q", F2.tobytes(), 32)[0]
    assert struct.unpack_from("<Q", D.tobytes(), 112)[0] == nch
    assert pbytes_d == pbytes_f and np.array_equal(D[poff_d:], F2[poff_f:])
    _check_delta_by_definition(D, F, F2, now, list(range(nch)))


def test_single_byte_change_marks_exactly_the_owning_chunk():
    rng = np.random.default_rng(23)
    combos = [c for k in (1, 2, 3) for c in itertools.product(SIZES, repeat=k)]
    combos = [c for i, c in enumerate(combos) if len(c) < 3 or i % 5 == 0]
    for c in combos:
        handles = sorted(rng.choice(np.arange(1, 500), size=len(c), replace=False).tolist())
        ents = [O.Entry(int(h), rng.integers(0, 256, s, dtype=np.uint8), int(h) * 3) for h, s in zip(handles, c)]
        nonempty = [i for i, s in enumerate(c) if s]
        if not nonempty:
            continue
        F = O.checkpoint(ents, device=1, epoch=5)
        i = int(rng.choice(nonempty))
        pos = int(rng.integers(0, c[i]))
        now = _mutate(ents, [(i, pos, int(rng.integers(1, 256)))])
        # owning chunk by FORMAT.md: chunks of the buffers before i, then pos // 65536
        k = sum((c[j] + 65535) // 65536 for j in range(len(c)) if handles[j] < handles[i]) + pos // 65536
        D = O.checkpoint_incremental(now, F, device=1, epoch=6)
        F2 = O.checkpoint(now, device=1, epoch=6)
        _check_delta_by_definition(D, F, F2, now, [k])
        st, M = O.merge(F, D)
        assert st == 0 and np.array_equal(M, F2)


def test_chain_of_deltas_merges_to_the_full_images():
    rng = np.random.default_rng(24)
    s0 = [O.Entry(h, rng.integers(0, 256, n, dtype=np.uint8)) for h, n in [(1, 300000), (2, 5), (3, 131072), (5, 70001)]]
    s1 = _mutate(s0, [(0, 70000, 1), (0, 299999, 2), (3, 3, 9)])
    s2 = _mutate(s1, [(2, 65536, 4), (1, 0, 1)])
    F0 = O.checkpoint(s0, epoch=0)
    D1 = O.checkpoint_incremental(s1, F0, epoch=1)
    D2 = O.checkpoint_incremental(s2, D1, epoch=2)  # a delta is the base of the next one
    st, M1 = O.merge(F0, D1)
    assert st == 0 and np.array_equal(M1, O.checkpoint(s1, epoch=1))
    st, M2 = O.merge(M1, D2)
    assert st == 0 and np.array_equal(M2, O.checkpoint(s2, epoch=2))
    st, rep, back = O.restore_chain([F0, D1, D2])
    assert st == 0
    for a, b in zip(back, s2):
        assert a.handle == b.handle and np.array_equal(a.data, b.data)
    # wrong link: D2 does not apply to F0 (base epoch and base table differ)
    assert O.merge(F0, D2)[0] == O.BAD_IMAGE
    # a delta alone is not a restorable image; a delta is not a merge base
    assert O.restore(D1)[0] == O.BAD_IMAGE
    assert O.merge(D1, D2)[0] == O.BAD_IMAGE


def test_layout_change_gives_the_full_image():
    rng = np.random.default_rng(25)
    s0 = [O.Entry(1, rng.integers(0, 256, 1000, dtype=np.uint8)), O.Entry(2, rng.integers(0, 256, 10, dtype=np.uint8))]
    F = O.checkpoint(s0, epoch=0)
    for now in (s0 + [O.Entry(3, np.ones(4, np.uint8))],                    # a buffer added
                s0[:1],                                                      # released
                [O.Entry(1, s0[0].data[:999]), s0[1]],                       # resized
                [O.Entry(1, s0[0].data, flags=7), s0[1]]):                   # flags changed
        D = O.checkpoint_incremental(now, F, epoch=1)
        assert np.array_equal(D, O.checkpoint(now, epoch=1))
    assert np.array_equal(O.checkpoint_incremental(s0, F, device=1, epoch=1), O.checkpoint(s0, device=1, epoch=1))


def test_delta_corruption_every_metadata_bit_and_payload_localisation():
    rng = np.random.default_rng(26)
    s0 = [O.Entry(2, rng.integers(0, 256, 70000, dtype=np.uint8)), O.Entry(6, rng.integers(0, 256, 33, dtype=np.uint8))]
    s1 = _mutate(s0, [(0, 65540, 0x10), (1, 32, 1)])
    F = O.checkpoint(s0, epoch=3)
    D = O.checkpoint_incremental(s1, F, epoch=4)
    poff = struct.unpack_from("<Q", D.tobytes(), 56)[0]
    for pos in range(poff):
        for bit in range(8):
            bad = D.copy()
            bad[pos] ^= 1 << bit
            assert O.validate(bad)[0] == O.BAD_IMAGE, (pos, bit)
    # payload: the merge goes through, the restore reports the chunk the span maps to
    spans = [(k, s, t) for k, s, t in _spans(s1) if k in (1, 2)]
    pos_in_delta = poff
    for k, s, t in spans:
        bad = D.copy()
        bad[pos_in_delta + (t - s) // 2] ^= 0x80
        st, M = O.merge(F, bad)
        assert st == 0
        st, rep, _ = O.restore(M)
        assert st == O.CRC_MISMATCH and rep["first_bad_chunk"] == k and rep["n_bad_chunks"] == 1
        pos_in_delta += t - s


def test_crc_blind_change_is_not_in_the_delta():
    """Reading 21 made visible: "updated" is decided by the CRC, so a change whose
    CRC difference is zero (a non-zero vector in the kernel of the GF(2)-linear map
    data -> CRC, found here by Gaussian elimination over 40 bits) is not written."""
    n = 64
    base = np.zeros(n, np.uint8)
    c0 = O.crc32c(base)
    cols = []
    for bit in range(40):
        e = base.copy()
        e[bit // 8] ^= 1 << (bit % 8)
        cols.append(O.crc32c(e) ^ c0)
    # find a non-empty subset of the 40 columns that XORs to 0 (GF(2) elimination)
    pivots = {}
    combo = None
    for i, v in enumerate(cols):
        mask = 1 << i
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
    assert combo
    delta_bytes = np.zeros(n, np.uint8)
    for bit in range(40):
        if combo >> bit & 1:
            delta_bytes[bit // 8] ^= 1 << (bit % 8)
    rng = np.random.default_rng(27)
    data = rng.integers(0, 256, n, dtype=np.uint8)
    assert O.crc32c(data ^ delta_bytes) == O.crc32c(data)
    F = O.checkpoint([O.Entry(1, data)], epoch=0)
    D = O.checkpoint_incremental([O.Entry(1, data ^ delta_bytes)], F, epoch=1)
    assert struct.unpack_from("<Q", D.tobytes(), 112)[0] == 0  # not present


# ---- dirty rule 1: a chunk is updated iff its bytes differ (reading 25) ----

def _crc_blind_delta(n=64):
    """A non-zero change vector whose CRC32C difference is zero (GF(2) elimination
    over the CRC's linear map restricted to the first 40 bits)."""
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
    d = np.zeros(n, np.uint8)
    for i in range(40):
        if combo >> i & 1:
            d[i // 8] ^= 1 << (i % 8)
    return d


def _byte_present(old_ents, new_ents):
    """Chunks whose bytes differ, by FORMAT.md's chunking, computed here with numpy."""
    out, k = [], 0
    for a, b in zip(sorted(old_ents, key=lambda e: e.handle), sorted(new_ents, key=lambda e: e.handle)):
        for j in range((a.data.size + 65535) // 65536):
            if not np.array_equal(a.data[65536 * j:65536 * (j + 1)], b.data[65536 * j:65536 * (j + 1)]):
                out.append(k)
            k += 1
    return out


def test_bytes_rule_writes_the_crc_blind_change():
    """The change the CRC rule misses (test_crc_blind_change_is_not_in_the_delta) is
    present under the bytes rule, and merge(F, D) is the full image of the new state,
    byte for byte; under the CRC rule the merge keeps the stale bytes."""
    d = _crc_blind_delta()
    rng = np.random.default_rng(31)
    data = rng.integers(0, 256, 70000, dtype=np.uint8)
    now = data.copy()
    now[65536:65536 + d.size] ^= d  # inside chunk 1
    assert O.crc32c(now[65536:]) == O.crc32c(data[65536:])
    F = O.checkpoint([O.Entry(1, data)], epoch=0)
    F2 = O.checkpoint([O.Entry(1, now)], epoch=1)
    D = O.checkpoint_incremental([O.Entry(1, now)], F, epoch=1, rule=O.RULE_BYTES, base_full=F)
    _check_delta_by_definition(D, F, F2, [O.Entry(1, now)], [1], rule=1)
    st, M = O.merge(F, D)
    assert st == 0 and np.array_equal(M, F2)
    Dc = O.checkpoint_incremental([O.Entry(1, now)], F, epoch=1, rule=O.RULE_CRC)
    st, Mc = O.merge(F, Dc)
    assert st == 0 and not np.array_equal(Mc, F2)  # the CRC rule's documented miss


def test_bytes_rule_present_set_is_the_byte_difference():
    rng = np.random.default_rng(32)
    for trial in range(40):
        sizes = [int(x) for x in rng.choice(SIZES + [200003, 1], size=int(rng.integers(1, 4)))]
        handles = sorted(rng.choice(np.arange(1, 100), size=len(sizes), replace=False).tolist())
        ents = [O.Entry(int(h), rng.integers(0, 256, s, dtype=np.uint8), trial) for h, s in zip(handles, sizes)]
        changes = []
        for i, s in enumerate(sizes):
            for _ in range(int(rng.integers(0, 4)) if s else 0):
                changes.append((i, int(rng.integers(0, s)), int(rng.integers(1, 256))))
        if changes and trial % 3 == 0:  # a change undone by a second one: bytes equal again
            i, pos, x = changes[0]
            changes.append((i, pos, x))
        now = _mutate(ents, changes)
        F = O.checkpoint(ents, device=3, epoch=trial)
        F2 = O.checkpoint(now, device=3, epoch=trial + 1)
        D = O.checkpoint_incremental(now, F, device=3, epoch=trial + 1, rule=O.RULE_BYTES, base_full=F)
        _check_delta_by_definition(D, F, F2, now, _byte_present(ents, now), rule=1)
        st, M = O.merge(F, D)
        assert st == 0 and np.array_equal(M, F2)


def test_bytes_rule_chain_with_delta_base():
    """A delta as the base: base_full is the merge of its chain."""
    rng = np.random.default_rng(33)
    s0 = [O.Entry(h, rng.integers(0, 256, n, dtype=np.uint8)) for h, n in [(1, 300000), (2, 5), (3, 131072)]]
    d = _crc_blind_delta()
    s1 = _mutate(s0, [(0, 70000, 1), (2, 3, 9)])
    s2 = [O.Entry(e.handle, e.data.copy(), e.flags) for e in s1]
    s2[0].data[131072:131072 + d.size] ^= d  # CRC-blind, in chunk 2 of buffer 1
    F0 = O.checkpoint(s0, epoch=0)
    D1 = O.checkpoint_incremental(s1, F0, epoch=1, rule=O.RULE_BYTES, base_full=F0)
    st, M1 = O.merge(F0, D1)
    assert st == 0
    D2 = O.checkpoint_incremental(s2, D1, epoch=2, rule=O.RULE_BYTES, base_full=M1)
    assert struct.unpack_from("<Q", D2.tobytes(), 112)[0] == 1
    st, rep, back = O.restore_chain([F0, D1, D2])
    assert st == 0 and all(np.array_equal(a.data, b.data) for a, b in zip(back, s2))
    st, M2 = O.merge(M1, D2)
    assert st == 0 and np.array_equal(M2, O.checkpoint(s2, epoch=2))


def test_bytes_rule_needs_the_base_state():
    rng = np.random.default_rng(34)
    s0 = [O.Entry(1, rng.integers(0, 256, 1000, dtype=np.uint8))]
    s1 = _mutate(s0, [(0, 5, 1)])
    F0 = O.checkpoint(s0, epoch=0)
    F1 = O.checkpoint(s1, epoch=1)
    with pytest.raises(ValueError):  # no base state
        O.checkpoint_incremental(s1, F0, epoch=2, rule=O.RULE_BYTES)
    with pytest.raises(ValueError):  # the state of another epoch
        O.checkpoint_incremental(s1, F0, epoch=2, rule=O.RULE_BYTES, base_full=F1)
    with pytest.raises(ValueError):  # no such rule
        O.checkpoint_incremental(s1, F0, epoch=2, rule=2, base_full=F0)


def test_dirty_rule_field_validation():
    """FORMAT.md: a delta's dirty_rule (offset 108) is 0 or 1; anything else is
    BAD_IMAGE even with a correct meta CRC (recomputed here with the hardware crc32)."""
    rng = np.random.default_rng(35)
    s0 = [O.Entry(1, rng.integers(0, 256, 100000, dtype=np.uint8))]
    F = O.checkpoint(s0, epoch=0)
    D = O.checkpoint_incremental(_mutate(s0, [(0, 1, 1)]), F, epoch=1, rule=O.RULE_BYTES, base_full=F)
    assert O.validate(D)[0] == 0 and struct.unpack_from("<I", D.tobytes(), 108)[0] == 1
    poff = struct.unpack_from("<Q", D.tobytes(), 56)[0]
    for v, want in ((0, 0), (2, O.BAD_IMAGE), (0xFFFFFFFF, O.BAD_IMAGE)):
        bad = bytearray(D.tobytes())
        struct.pack_into("<I", bad, 108, v)
        struct.pack_into("<I", bad, 124, _crc(bytes(bad[:124]) + bytes(bad[128:poff])))
        assert O.validate(np.frombuffer(bytes(bad), np.uint8))[0] == want, v
