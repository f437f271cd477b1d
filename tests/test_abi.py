"""-m "not gpu": the C-ABI library loads, exports every symbol include/checl.h
declares, and its host logic (handle table, overlap checks, ids, wrapped images,
status strings) works from C and from Python without a GPU."""
import os
import re
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "checl.h")
PKG = os.path.join(ROOT, "paper_conf_ipps_takizawakskk11_b200")
LIB = os.path.join(PKG, "libchecl.so")


@pytest.fixture(scope="module")
def built():
    from paper_conf_ipps_takizawakskk11_b200 import build
    build.build()
    return LIB


def declared_symbols():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(checl_[a-z_]+)\s*\(", text)))


def test_header_declares_the_north_star_calls():
    syms = declared_symbols()
    for s in ("checl_register_buffer", "checl_release", "checl_checkpoint", "checl_restore", "checl_translate",
              "checl_migrate", "checl_image_free"):
        assert s in syms


def test_library_exports_every_declared_symbol(built):
    out = subprocess.run(["nm", "-D", "--defined-only", built], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (checl_\w+)", out))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, missing


def test_library_is_sm100a(built):
    out = subprocess.run(["cuobjdump", "--list-elf", built], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_product_library_has_no_experiment_hooks(built):
    """The A/B and tracing switches live only in the experiments build
    (libchecl_exp.so, -DCHECL_EXPERIMENTS): the product library does not even contain
    their names, so no environment variable can turn a checkpoint into an invalid
    image or add tracing to the hot path."""
    data = open(built, "rb").read()
    for name in (b"CHECL_EXP_PACK_OP", b"CHECL_WARP_TRACE", b"CHECL_STAGE_TRACE", b"CHECL_TABLE_MC",
                 b"CHECL_STATIC_PERMILLE", b"CHECL_DYN_BLOCK", b"CHECL_D2H_SPLIT"):
        assert name not in data, name
    from paper_conf_ipps_takizawakskk11_b200 import build
    build.build(experiments=True)
    assert b"CHECL_EXP_PACK_OP" in open(build.LIB_EXP, "rb").read()


def test_python_binding_declares_every_export(built):
    from paper_conf_ipps_takizawakskk11_b200 import checl
    assert sorted(checl.EXPORTS) == declared_symbols()
    for s in checl.EXPORTS:
        assert hasattr(checl.lib, s)


def test_c_client_registry_without_gpu(built, tmp_path):
    exe = tmp_path / "abi_registry"
    subprocess.check_call(["gcc", "-std=c99", "-Wall", "-Werror", f"-I{ROOT}/include",
                           os.path.join(ROOT, "tests", "c", "abi_registry.c"), f"-L{PKG}", "-lchecl",
                           f"-Wl,-rpath,{PKG}", "-o", str(exe)])
    env = dict(os.environ, CHECL_FAKE_DEVICES="2")
    r = subprocess.run([str(exe)], capture_output=True, text=True, env=env)
    assert r.returncode == 0, r.stderr
    assert "abi_registry ok" in r.stdout


PY_REGISTRY = r"""
import os, sys
sys.path.insert(0, %r)
from paper_conf_ipps_takizawakskk11_b200 import checl
c = checl.Context(allocator="cuda")
hs = [c.register_ptr(0, 0x10000 + 0x1000 * i, 0x800 + i, flags=i) for i in range(100)]
assert hs == list(range(1, 101))
assert c.count(0) == (100, sum(0x800 + i for i in range(100)))
for h in hs[::2]:
    c.release(h)
assert c.count(0)[0] == 50
assert c.translate(hs[1]) == (0x11000, 0x801, 0)
try:
    c.register_ptr(0, 0x11000 + 0x800, 4)
    raise SystemExit("overlap not detected")
except checl.CheclError as e:
    assert e.status == checl.ERR_INVALID_VALUE
assert c.register_ptr(0, 0x10000, 0x1000) == 101   # released range reusable, id fresh
img = checl.Image.wrap(bytes(4096))
assert img.view().size == 4096 and img.info()["location"] == checl.IMAGE_HOST
try:  # an unknown dirty rule is refused before any device work
    c.checkpoint_incremental(0, img, epoch=1, rule=7)
    raise SystemExit("unknown dirty rule accepted")
except checl.CheclError as e:
    assert e.status == checl.ERR_INVALID_VALUE
img.free()
c.trim()  # nothing kept yet: a no-op without a device
c.close()
print("ok")
"""


def test_python_registry_without_gpu(built):
    env = dict(os.environ, CHECL_FAKE_DEVICES="1")
    r = subprocess.run([sys.executable, "-c", PY_REGISTRY % ROOT], capture_output=True, text=True, env=env)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr


def test_missing_library_fails_loudly(tmp_path):
    # a copy of the package without libchecl.so must refuse to import (no CPU fallback)
    import shutil
    dst = tmp_path / "paper_conf_ipps_takizawakskk11_b200"
    shutil.copytree(PKG, dst, ignore=shutil.ignore_patterns("*.so", "build_obj*", "__pycache__"))
    r = subprocess.run([sys.executable, "-c", "import paper_conf_ipps_takizawakskk11_b200"], cwd=tmp_path,
                       capture_output=True, text=True)
    assert r.returncode != 0 and "ImportError" in r.stderr and "no CPU fallback" in r.stderr


PY_HOST_PATHS = r"""
import os, signal, sys, struct
sys.path.insert(0, %r)
import numpy as np
from paper_conf_ipps_takizawakskk11_b200 import checl
from oracle import oracle as O
tmp = sys.argv[1]

# delayed checkpointing mode (L16): the signal only marks the request
c = checl.Context(allocator="cuda")
assert not c.checkpoint_pending()
c.install_signal(signal.SIGUSR1)
os.kill(os.getpid(), signal.SIGUSR1)
assert c.checkpoint_pending()
c2 = checl.Context(allocator="cuda")
assert not c2.checkpoint_pending()
c2.request_checkpoint()
assert c2.checkpoint_pending()
try:
    c.install_signal(signal.SIGKILL)
    raise SystemExit("SIGKILL accepted")
except checl.CheclError as e:
    assert e.status == checl.ERR_INVALID_VALUE
c.close()   # unregisters its handler binding
os.kill(os.getpid(), signal.SIGUSR1)   # handler sees no context: ignored
c2.close()

# writing phase: oracle images (full and incremental) through write/read, both I/O modes
rng = np.random.default_rng(1)
ents = [O.Entry(1, rng.integers(0, 256, 300001, dtype=np.uint8)), O.Entry(4, rng.integers(0, 256, 13, dtype=np.uint8))]
full = O.checkpoint(ents, device=0, epoch=7)
ents[0].data[100000] ^= 1
delta = O.checkpoint_incremental(ents, full, device=0, epoch=8)
for name, arr in (("full", full), ("delta", delta)):
    for direct in (True, False):
        img = checl.Image.wrap(arr)
        path = os.path.join(tmp, f"{name}{int(direct)}.checl")
        img.write(path, direct=direct, sync=True)
        assert os.path.getsize(path) == arr.size
        back = checl.Image.read(path, direct=direct)
        assert np.array_equal(back.view(), arr)
        assert back.header()["flags"] == (1 if name == "delta" else 0)
        back.free(); img.free()
# library merge of the re-read images == oracle merge
F = checl.Image.read(os.path.join(tmp, "full1.checl"))
D = checl.Image.read(os.path.join(tmp, "delta1.checl"))
st, want = O.merge(full, delta)
assert st == 0 and np.array_equal(F.merge(D).view(), want)
# a view keeps its image alive (the merged image above is a temporary)
import gc, weakref
m = F.merge(D)
w = weakref.ref(m)
v = m.view()
del m
gc.collect()
assert w() is not None and np.array_equal(v, want)
del v
gc.collect()
assert w() is None
# a delta of the exact (bytes) dirty rule parses and merges in the library like the
# oracle's (FORMAT.md dirty_rule = 1); an unknown rule value is BAD_IMAGE
delta_b = O.checkpoint_incremental(ents, full, device=0, epoch=8, rule=O.RULE_BYTES, base_full=full)
st, want_b = O.merge(full, delta_b)
Db = checl.Image.wrap(delta_b)
assert st == 0 and Db.header()["dirty_rule"] == 1 and np.array_equal(F.merge(Db).view(), want_b)
bad_rule = bytearray(delta_b.tobytes())
struct.pack_into("<I", bad_rule, 108, 2)
poff = struct.unpack_from("<Q", bad_rule, 56)[0]
struct.pack_into("<I", bad_rule, 124, O.crc32c(bytes(bad_rule[:124]) + bytes(bad_rule[128:poff])))
try:
    F.merge(checl.Image.wrap(np.frombuffer(bytes(bad_rule), np.uint8)))
    raise SystemExit("dirty_rule 2 accepted")
except checl.CheclError as e:
    assert e.status == checl.ERR_BAD_IMAGE
# damaged files are refused at read
p = os.path.join(tmp, "full1.checl")
raw = bytearray(open(p, "rb").read())
for bad in (raw[:-1], raw[:100], raw[:40] + bytes([raw[40] ^ 1]) + raw[41:]):
    q = os.path.join(tmp, "bad.checl")
    open(q, "wb").write(bytes(bad))
    try:
        checl.Image.read(q)
        raise SystemExit("damaged image accepted")
    except checl.CheclError as e:
        assert e.status == checl.ERR_BAD_IMAGE, e
# host meta CRC (3 interleaved crc32 streams over 3 KiB blocks + a tail) on metadata
# of 0.2-60 KB: every oracle image is accepted, a flipped metadata bit is refused
for nb in (1, 20, 63, 64, 65, 200, 1000):
    ents = [O.Entry(i + 1, rng.integers(0, 256, int(rng.integers(0, 3 * 65536)), dtype=np.uint8)) for i in range(nb)]
    arr = O.checkpoint(ents, device=0, epoch=nb)
    q = os.path.join(tmp, "meta.checl")
    w = checl.Image.wrap(arr)
    w.write(q)
    back = checl.Image.read(q)
    assert np.array_equal(back.view(), arr)
    back.free(); w.free()
    poff = struct.unpack_from("<Q", arr.tobytes(), 56)[0]
    for pos in (130, poff // 2, poff - 1 if nb == 1 else int(poff) - 8):
        bad = arr.copy()
        bad[pos] ^= 0x20
        open(q, "wb").write(bad.tobytes())
        try:
            checl.Image.read(q)
            raise SystemExit(f"metadata flip at {pos} accepted (nb={nb})")
        except checl.CheclError as e:
            assert e.status == checl.ERR_BAD_IMAGE, e
print("ok")
"""


def test_delayed_mode_signal_and_image_files_without_gpu(built, tmp_path):
    env = dict(os.environ, CHECL_FAKE_DEVICES="1")
    r = subprocess.run([sys.executable, "-c", PY_HOST_PATHS % ROOT, str(tmp_path)], capture_output=True, text=True,
                       env=env, cwd=ROOT)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout + r.stderr
