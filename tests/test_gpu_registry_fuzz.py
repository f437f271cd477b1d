"""-m gpu: seeded random sequences of registry and snapshot calls against a model.

The restore fast paths (cached layout, chunk-list keys, in-place rebinding through a
binding, spare segments) remember state across calls. This test drives a
context through random interleavings — register, release, write into live buffers,
checkpoint to host / HBM images, restore an image (the latest or an older one, host or
device), migrate in place, incremental checkpoint + chain restore — and after every call
checks every live handle against a Python model: its size and device (translate) and its
bytes (the image contents it was restored from, or the user's writes). The model
follows PAPER.md L15 (handles stay valid, translation gives the current buffer) and
FORMAT.md (an image restores exactly the bytes it was taken with)."""
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

DEV = 0


def _bytes(ctx, h):
    ptr, nb, dev = ctx.translate(h)
    if nb == 0:
        return np.zeros(0, np.uint8)
    return ctx.tensor(h).cpu().numpy()


# CHECL_REG_FUZZ_CASES widens the sweep (default 16 sequences of 60 calls)
@pytest.mark.parametrize("seed", range(int(os.environ.get("CHECL_REG_FUZZ_CASES", "16"))))
def test_random_call_sequences_match_model(seed):
    rng = np.random.default_rng(900 + seed)
    ctx = checl.Context()
    if seed % 3 == 1:
        ctx.set_staging(65536 * 3, 2)
    model = {}     # handle -> expected bytes (np.uint8)
    keep = {}      # handle -> the user tensor backing a user registration (kept alive)
    images = []    # (Image, {handle: bytes} at checkpoint time)

    def new_buffer():
        size = int(rng.choice([0, 1, 17, 4097, 65536, 65537, 200_003, int(rng.integers(1, 1 << 20))]))
        t = torch.empty(size + 16, dtype=torch.uint8, device=DEV)
        off = int(rng.integers(0, 8))
        v = t[off:off + size]
        if size:
            checl.debug_fill(v, int(rng.integers(0, 1 << 30)), 0)
        torch.cuda.synchronize()
        h = ctx.register(v, int(rng.integers(0, 4)))
        keep[h] = t
        model[h] = v.cpu().numpy().copy()

    def check(step, what):
        for h, want in model.items():
            ptr, nb, dev = ctx.translate(h)
            assert (nb, dev) == (want.size, DEV), (step, what, h)
            assert np.array_equal(_bytes(ctx, h), want), (step, what, h)
        n, _ = ctx.count(DEV)
        assert n == len(model), (step, what)

    for _ in range(4):
        new_buffer()
    for step in range(60):
        op = rng.choice(["reg", "rel", "write", "ckpt", "ckpt_dev", "restore", "restore_again", "migrate", "incr"],
                        p=[.1, .08, .16, .12, .1, .18, .12, .06, .08])
        if op == "reg" or not model:
            new_buffer()
        elif op == "rel":
            h = int(rng.choice(list(model)))
            ctx.release(h)
            del model[h]
            keep.pop(h, None)
        elif op == "write":
            hs = [h for h in model if model[h].size]
            if hs:
                h = int(rng.choice(hs))
                pos = int(rng.integers(0, model[h].size))
                ctx.tensor(h)[pos:pos + 1].bitwise_xor_(0x5A)
                torch.cuda.synchronize()
                model[h][pos] ^= 0x5A
        elif op in ("ckpt", "ckpt_dev"):
            img = ctx.checkpoint(DEV, epoch=step) if op == "ckpt" else ctx.checkpoint_device(DEV, epoch=step)
            images.append((img, {h: b.copy() for h, b in model.items()}))
            if len(images) > 4:
                images.pop(0)[0].free()
        elif op in ("restore", "restore_again") and images:
            img, state = images[-1] if op == "restore_again" else images[int(rng.integers(0, len(images)))]
            rep = ctx.restore(img, DEV)
            assert rep.n_bad_chunks == 0
            for h, b in state.items():
                model[h] = b.copy()
                keep.pop(h, None)  # now library-owned
        elif op == "migrate":
            ctx.migrate(DEV, DEV)
            keep.clear()  # every live buffer is now library-owned
        elif op == "incr" and images:
            base, state = images[-1]
            if base.info()["location"] == checl.IMAGE_HOST:
                rule = checl.DIRTY_BYTES if step % 2 else checl.DIRTY_CRC
                d = ctx.checkpoint_incremental(DEV, base, epoch=step, rule=rule)
                if d.header()["flags"] == 1:
                    now = {h: b.copy() for h, b in model.items()}
                    rep = ctx.restore_chain([base, d], DEV)
                    assert rep.n_bad_chunks == 0
                    for h, b in now.items():
                        model[h] = b
                        keep.pop(h, None)
                d.free()
        check(step, op)
    for img, _ in images:
        img.free()
    ctx.close()
