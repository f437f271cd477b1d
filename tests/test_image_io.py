"""-m "not gpu": the writing phase (checl_image_write; PAPER.md
L16 §III-C checkpoint step 3, Table I) reports a full disk as an error.

A host image is written through a shared mapping of the file when O_DIRECT does not
apply (tmpfs, pageable or unaligned images). A page fault of a mapping that finds the
file system full raises SIGBUS instead of returning an error, so the library reserves
the file's blocks first and falls back to pwrite when it cannot. These tests run the
write in a child process on a 1 MiB tmpfs: the child must survive and report
CHECL_ERR_INVALID_VALUE (checl.h), and an image that fits must round-trip."""
import os
import subprocess
import sys
import uuid

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys
sys.path.insert(0, %(root)r)
import numpy as np
import synth
from oracle import oracle as O
from paper_conf_ipps_takizawakskk11_b200 import checl
size = %(size)d
img = O.checkpoint([O.Entry(1, synth.fill_bytes(size, 3, 0), 0)], device=0, epoch=1)
buf = np.empty(img.size + 1, dtype=np.uint8)[1:]  # (unaligned: never O_DIRECT)
buf[:] = img
w = checl.Image.wrap(buf)
try:
    w.write(%(path)r, direct=%(direct)r)
except checl.CheclError as e:
    print("status", e.status)
    raise SystemExit(0)
back = checl.Image.read(%(path)r, direct=False)
print("status 0", int(np.array_equal(back.view(), img)))
"""


@pytest.fixture()
def small_tmpfs(tmp_path):
    mnt = tmp_path / "fs"
    mnt.mkdir()
    r = subprocess.run(["mount", "-t", "tmpfs", "-o", "size=1m", "tmpfs", str(mnt)], capture_output=True)
    if r.returncode != 0:
        pytest.skip("cannot mount a small tmpfs here")
    yield str(mnt)
    subprocess.run(["umount", str(mnt)], capture_output=True)


def _child(path: str, size: int, direct: bool):
    code = CHILD % {"root": ROOT, "size": size, "path": path, "direct": direct}
    return subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, cwd=ROOT, timeout=120,
                          env=dict(os.environ, CUDA_VISIBLE_DEVICES=""))


@pytest.mark.parametrize("direct", [False, True])
def test_write_to_full_filesystem_returns_error_not_sigbus(small_tmpfs, direct):
    r = _child(os.path.join(small_tmpfs, f"img-{uuid.uuid4().hex}"), 3 << 20, direct)
    assert r.returncode == 0, f"child died with {r.returncode}: {r.stderr[-2000:]}"
    assert "status -1" in r.stdout, r.stdout + r.stderr


def test_write_that_fits_round_trips(small_tmpfs):
    r = _child(os.path.join(small_tmpfs, "img"), 300_000, False)
    assert r.returncode == 0, r.stderr[-2000:]
    assert "status 0 1" in r.stdout, r.stdout + r.stderr
