"""-m gpu: configs[3] (C4, SHOC-MD-shaped rank, 64 GiB) at full size on one B200.

Checkpoint to a pinned host image, then restore into re-created buffers; the image
header/manifest/CRC table are checked against the oracle's layout and meta CRC;
EVERY one of the 1,048,578 CRC-table entries against the x86 SSE4.2 crc32
instruction's CRC32C of its chunk (tests/helpers: independent of the oracle and of
the product, fast enough for 64 GiB), the whole payload against the buffers' bytes
read back with plain copies, and sampled chunks (random ones plus every buffer's
short tail chunk) against the oracle's CRC32C and the synth generator's bytes;
restored buffers are compared on the same samples.
"""
from concurrent.futures import ThreadPoolExecutor

import struct

import numpy as np
import pytest

import synth
from oracle import oracle as O

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402
from tests.helpers import hwcrc  # noqa: E402

PIECE = 1 << 30  # bytes per host piece (a multiple of the 64 KiB chunk)


def _chunk_crcs(host: np.ndarray, n: int) -> np.ndarray:
    """CRC32C (SSE4.2) of the 64 KiB chunks of host[:n], 8 threads."""
    offs = np.arange(0, n, 65536, dtype=np.uint64)
    lens = np.minimum(65536, n - offs).astype(np.uint64)
    parts = np.array_split(np.arange(offs.size), 8)
    with ThreadPoolExecutor(8) as ex:
        res = list(ex.map(lambda ix: hwcrc.hw_crc32c_many(host, offs[ix], lens[ix]), parts))
    return np.concatenate(res) if res else np.zeros(0, np.uint32)


def _full_table_and_payload_check(recs, crcs, dev_bytes_of, img_payload_of):
    """Every CRC entry = hw CRC32C of its chunk of the buffer's bytes (read back with a
    plain copy, dev_bytes_of(bi, lo, n)); with img_payload_of, the image's payload of
    every buffer equals those bytes."""
    for bi, (h, size, off, first, fl, dv, _) in enumerate(recs):
        for lo in range(0, size, PIECE):
            n = min(PIECE, size - lo)
            data = dev_bytes_of(bi, lo, n)
            hw = _chunk_crcs(data, n)
            k0 = first + lo // 65536
            assert np.array_equal(hw, crcs[k0:k0 + hw.size]), (bi, lo, int(np.count_nonzero(hw != crcs[k0:k0 + hw.size])))
            if img_payload_of is not None:
                assert np.array_equal(img_payload_of(off + lo, n), data), (bi, lo)


def test_c4_md_rank_full_size():
    w = synth.c4_md_rank(0)
    S = w.total_bytes
    free, _ = torch.cuda.mem_get_info(0)
    if free < S + (8 << 30):
        pytest.skip(f"needs {S >> 30} GiB free on the device")
    ctx = checl.Context()
    tensors = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
    for t, b in zip(tensors, w.buffers):
        checl.debug_fill(t, w.seed, b.stream, checl.FILL_FLOAT if b.name != "md.neigh" else checl.FILL_RANDOM)
    kinds = ["float" if b.name != "md.neigh" else "random" for b in w.buffers]
    torch.cuda.synchronize()
    handles = [ctx.register(t, 0x40 + i) for i, t in enumerate(tensors)]
    img = ctx.checkpoint(0, epoch=4)
    got = img.view()
    L = O.layout(list(zip(handles, [b.size for b in w.buffers])))
    assert got.size == L["image_bytes"] and L["payload_bytes"] == S + 288  # two 144-B alignment gaps
    assert L["n_chunks"] == 1048578
    st, rep = O.validate(got)  # header, manifest, meta CRC over the 4 MiB CRC table
    assert st == 0 and rep["n_chunks"] == 1048578
    recs = [struct.unpack_from("<QQQQIiQ", got, 128 + 48 * i) for i in range(3)]
    crcs = np.frombuffer(got, dtype="<u4", count=L["n_chunks"], offset=L["crc_off"])
    if hwcrc.available():
        _full_table_and_payload_check(
            recs, crcs, lambda bi, lo, n: tensors[bi][lo:lo + n].cpu().numpy(),
            lambda o, n: got[L["payload_off"] + o:L["payload_off"] + o + n])
    rng = np.random.default_rng(44)
    samples = []
    for bi, (h, size, off, first, fl, dv, _) in enumerate(recs):
        nch = (size + 65535) // 65536
        ks = list(rng.integers(0, nch, 12)) + [nch - 1]
        samples += [(bi, int(k)) for k in ks]
    for bi, k in samples:
        h, size, off, first, fl, dv, _ = recs[bi]
        lo = k * 65536
        n = min(65536, size - lo)
        data = synth.fill_slice(lo, n, w.seed, w.buffers[bi].stream, kinds[bi])
        p0 = L["payload_off"] + off + lo
        assert np.array_equal(got[p0:p0 + n], data), (bi, k)
        assert int(crcs[first + k]) == O.crc32c(data), (bi, k)
    del tensors
    torch.cuda.empty_cache()
    rep = ctx.restore(img, 0)
    assert rep.n_bad_chunks == 0 and rep.n_chunks == 1048578
    for bi, k in samples:
        lo = k * 65536
        n = min(65536, w.buffers[bi].size - lo)
        back = ctx.tensor(handles[bi])[lo:lo + n].cpu().numpy()
        assert np.array_equal(back, synth.fill_slice(lo, n, w.seed, w.buffers[bi].stream, kinds[bi])), (bi, k)
    img.free()
    ctx.close()


def _device_bytes(ptr: int, n: int) -> np.ndarray:
    """n bytes of device memory at ptr (a torch view, copied to the host)."""
    class _Iface:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (ptr, False), "version": 2,
                                    "strides": None}
    return torch.as_tensor(_Iface(), device="cuda:0").cpu().numpy()


def test_c4_full_size_device_image_restart():
    """configs[3] at full size in bench.py's launch configuration: HBM-resident image,
    restart mode (every handle released, restore re-creates the buffers). The image
    metadata mirror, sampled CRC table entries and payload chunks are checked against
    the oracle's layout / CRC32C and the synth generator; the re-created buffers on the
    same samples."""
    w = synth.c4_md_rank(0)
    S = w.total_bytes
    torch.cuda.empty_cache()  # what an earlier test's restore left in torch's cache
    free, _ = torch.cuda.mem_get_info(0)
    if free < 2 * S + (8 << 30):
        pytest.skip(f"needs {2 * S >> 30} GiB free on the device")
    ctx = checl.Context()
    tensors = [torch.empty(b.size, dtype=torch.uint8, device=0) for b in w.buffers]
    for t, b in zip(tensors, w.buffers):
        checl.debug_fill(t, w.seed, b.stream, checl.FILL_RANDOM)
    torch.cuda.synchronize()
    handles = [ctx.register(t, 0x80 + i) for i, t in enumerate(tensors)]
    img = ctx.checkpoint_device(0, epoch=9)
    meta = np.array(img.view())
    hd = img.header()
    L = O.layout(list(zip(handles, [b.size for b in w.buffers])))
    assert meta.size == L["payload_off"] and hd["image_bytes"] == L["image_bytes"]
    assert (hd["n_buffers"], hd["n_chunks"], hd["crc_off"], hd["payload_bytes"], hd["epoch"]) == (
        3, L["n_chunks"], L["crc_off"], L["payload_bytes"], 9)
    recs = [struct.unpack_from("<QQQQIiQ", meta, 128 + 48 * i) for i in range(3)]
    crcs = np.frombuffer(meta, dtype="<u4", count=L["n_chunks"], offset=L["crc_off"])
    pay = img.info()["device_payload"]
    if hwcrc.available():
        # the whole CRC table against the buffers; the HBM payload against them on the
        # device (torch.equal: a plain comparison, not the library's)
        _full_table_and_payload_check(recs, crcs, lambda bi, lo, n: tensors[bi][lo:lo + n].cpu().numpy(), None)
        for bi, (h, size, off, first, fl, dv, _) in enumerate(recs):
            for lo in range(0, size, PIECE):
                n = min(PIECE, size - lo)
                class _I:
                    __cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (pay + off + lo, False),
                                                "version": 2, "strides": None}
                assert torch.equal(torch.as_tensor(_I(), device="cuda:0"), tensors[bi][lo:lo + n]), (bi, lo)
    rng = np.random.default_rng(45)
    samples = []
    for bi, (h, size, off, first, fl, dv, _) in enumerate(recs):
        assert (h, size, fl, dv) == (handles[bi], w.buffers[bi].size, 0x80 + bi, 0)
        nch = (size + 65535) // 65536
        samples += [(bi, int(k)) for k in list(rng.integers(0, nch, 10)) + [0, nch - 1]]
    for bi, k in samples:
        h, size, off, first, fl, dv, _ = recs[bi]
        lo = k * 65536
        n = min(65536, size - lo)
        data = synth.fill_slice(lo, n, w.seed, w.buffers[bi].stream, "random")
        assert np.array_equal(_device_bytes(pay + off + lo, n), data), (bi, k)
        assert int(crcs[first + k]) == O.crc32c(data), (bi, k)
    # restart: the application's buffers are gone, restore re-creates every handle
    for h in handles:
        ctx.release(h)
    del tensors, t
    torch.cuda.empty_cache()
    rep = ctx.restore(img, 0)
    assert rep.n_bad_chunks == 0 and rep.n_chunks == L["n_chunks"] and rep.n_buffers == 3
    for bi, k in samples:
        lo = k * 65536
        n = min(65536, w.buffers[bi].size - lo)
        back = ctx.tensor(handles[bi])[lo:lo + n].cpu().numpy()
        assert np.array_equal(back, synth.fill_slice(lo, n, w.seed, w.buffers[bi].stream, "random")), (bi, k)
        assert ctx.translate(handles[bi])[1:] == (w.buffers[bi].size, 0)
    img.free()
    ctx.close()
