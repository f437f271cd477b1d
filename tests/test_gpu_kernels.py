"""-m gpu: every kernel shape of the data path produces the same bytes.

libchecl dispatches a launch to one of four kernels: 1 grid-stride
warp per chunk, 2 grid-stride 4 KiB units, 3 balanced stretches of rounds (partial
chunks combined through the atomic CRC accumulator), 4 the same split with bulk
(TMA) copies, the column CRC and a dynamic tail. CHECL_KERNEL=k forces one;
each run here (a subprocess: the choice is read once per device) checkpoints a
registry with ragged, misaligned, multi-chunk and zero-size buffers, in one launch
and through small staging slots, compares the image with the oracle byte for byte,
restores it (host and HBM images) and checks the restored bytes."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import sys
sys.path.insert(0, %r)
import numpy as np, torch
from oracle import oracle as O
from tests.gpu_util import make_set, oracle_entries, bound_bytes
from paper_conf_ipps_takizawakskk11_b200 import checl
sizes = [1 << 20, 0, 65536 * 3 + 17, 4097, 1, 300007, 65535, 65537, 2 << 20]
for slot in (None, 196608):
    ctx = checl.Context()
    if slot:
        ctx.set_staging(slot, 2)
    ds = make_set(ctx, sizes, seed=21, offsets=[0, 0, 1, 4, 0, 8, 3, 0, 0])
    want = O.checkpoint(oracle_entries(ds), device=0, epoch=3)
    img = ctx.checkpoint(0, epoch=3)
    assert np.array_equal(img.view(), want), "host image"
    dimg = ctx.checkpoint_device(0, epoch=3)
    assert np.array_equal(dimg.view(), want[:dimg.view().size]), "device image metadata"
    for im in (img, dimg):
        for t in ds.tensors:
            t.zero_()
        rep = ctx.restore(im, 0)
        assert rep.n_bad_chunks == 0
        for h, b in zip(ds.handles, ds.host):
            assert np.array_equal(bound_bytes(ctx, h), b)
    rep = ctx.migrate(0, 0)  # K1 into an HBM image, K2 from it (peer path / fallback per env)
    assert rep.n_bad_chunks == 0
    for h, b in zip(ds.handles, ds.host):
        assert np.array_equal(bound_bytes(ctx, h), b), "migrate"
    bad = img.view().copy()
    poff = int(img.header()["payload_off"])
    bad[poff + 65536 * 16 + 5] ^= 1
    st, rep_o, _ = O.restore(bad)
    try:
        ctx.restore(checl.Image.wrap(bad), 0)
        raise SystemExit("corruption not detected")
    except checl.CheclError as e:
        assert e.report.first_bad_chunk == rep_o["first_bad_chunk"]
    # a corrupted HBM image (K2 reads it in place; with CHECL_FORCE_IMAGE_REMOTE as a peer's)
    dimg.corrupt(poff + 65536 * 16 + 5, 1)
    try:
        ctx.restore(dimg, 0)
        raise SystemExit("device image corruption not detected")
    except checl.CheclError as e:
        assert e.report.first_bad_chunk == rep_o["first_bad_chunk"] and e.report.n_bad_chunks == 1
    ctx.close()
print("kernel ok")
"""


@pytest.mark.parametrize("kernel", ["1", "2", "3", "4", "4:0:1", "4:500:3", "4:900:16", "4:0:1:mc", "4:500:3:mc",
                                    "0:remote", "4:remote", "4:0:1:remote", "0:nopeer", "4:nopeer", "0:nozc",
                                    "4:peerbulk"])
def test_forced_kernel_shapes_bit_exact(kernel):
    """kernel "4:S:B" = the TMA kernel with the dynamic tail forced on at this size:
    static share S permille, dynamic blocks of B rounds (S = 0: every round dynamic;
    with ":mc" the grid is rounded down to whole 2-CTA clusters, so the 3-chunk stages
    have more blocks than warps: every warp must keep fetching). ":remote": restores
    from the HBM image read it as a peer GPU's image (the migration i -> j path, which a
    one-GPU box cannot reach otherwise); ":nopeer": the fallback when peer access is
    unavailable (cudaMemcpyPeerAsync of the image, then K2 on the copy); ":nozc": small
    host images staged through a slot instead of the mapped pinned image; kernel "0" =
    the default dispatch."""
    k, *dyn = kernel.split(":")
    env = dict(os.environ, CHECL_KERNEL=k)
    if dyn and dyn[-1] == "peerbulk":  # the peer path with bulk copies (experiments build, CHECL_PEER_BULK)
        env.update(CHECL_FORCE_IMAGE_REMOTE="1", CHECL_PEER_BULK="1",
                   CHECL_LIB=os.path.join(ROOT, "paper_conf_ipps_takizawakskk11_b200", "libchecl_exp.so"))
        dyn = dyn[:-1]
    if dyn and dyn[-1] == "remote":  # K2 on an HBM image takes the peer-GPU read path (migration i -> j)
        env.update(CHECL_FORCE_IMAGE_REMOTE="1")
        dyn = dyn[:-1]
    if dyn and dyn[-1] == "nozc":  # small host images through the staging slot, not zero copy
        env.update(CHECL_ZERO_COPY_MAX="0")
        dyn = dyn[:-1]
    if dyn and dyn[-1] == "nopeer":  # no peer access: the image is copied to a local buffer first
        env.update(CHECL_FORCE_NO_PEER="1")
        dyn = dyn[:-1]
    if dyn and dyn[-1] == "mc":  # 2-CTA clusters with the multicast table prologue (even grids)
        env.update(CHECL_TABLE_MC="1")
        dyn = dyn[:-1]
    if dyn:
        env.update(CHECL_STATIC_PERMILLE=dyn[0], CHECL_DYN_BLOCK=dyn[1], CHECL_DYN_MIN_ROUNDS="0")
    if dyn or "CHECL_TABLE_MC" in env:  # those overrides exist only in the experiments build
        env.update(CHECL_LIB=os.path.join(ROOT, "paper_conf_ipps_takizawakskk11_b200", "libchecl_exp.so"))
    r = subprocess.run([sys.executable, "-c", SCRIPT % ROOT], capture_output=True, text=True, env=env, cwd=ROOT,
                       timeout=600)
    assert r.returncode == 0 and "kernel ok" in r.stdout, r.stdout + r.stderr


def test_product_build_ignores_experiment_hooks():
    """The product library does not read the experiments build's A/B switches: with
    CHECL_EXP_PACK_OP=2 (CRC-only pack, no valid image, in libchecl_exp.so) and the
    dynamic-tail overrides set, libchecl.so still writes the oracle's image."""
    env = dict(os.environ, CHECL_EXP_PACK_OP="2", CHECL_STATIC_PERMILLE="0", CHECL_DYN_BLOCK="1",
               CHECL_DYN_MIN_ROUNDS="0", CHECL_TABLE_MC="1", CHECL_WARP_TRACE="1")
    env.pop("CHECL_LIB", None)
    r = subprocess.run([sys.executable, "-c", SCRIPT % ROOT], capture_output=True, text=True, env=env, cwd=ROOT,
                       timeout=600)
    assert r.returncode == 0 and "kernel ok" in r.stdout, r.stdout + r.stderr
    assert "[checl] op" not in r.stderr  # no warp trace from the product library
