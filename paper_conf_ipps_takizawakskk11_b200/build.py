"""Builds libchecl.so in-tree (nvcc, sm_100a only).

    python -m paper_conf_ipps_takizawakskk11_b200.build [--force] [--exp]
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.environ.get("CHECL_LIB_OUT", os.path.join(PKG, "libchecl.so"))
# the experiments build (-DCHECL_EXPERIMENTS): the same sources plus the A/B and
# tracing hooks (CHECL_EXP_PACK_OP, warp/stage traces, dynamic-tail overrides, the
# multicast table prologue). Not the product: only tools/ and the kernel-shape tests
# that force those paths load it (CHECL_LIB=.../libchecl_exp.so).
LIB_EXP = os.path.join(PKG, "libchecl_exp.so")
EXTRA = os.environ.get("CHECL_EXTRA_FLAGS", "").split()  # experiments only (e.g. -DCHECL_WARPS=8)
SOURCES = ["checl_kernels.cu", "checl_engine.cpp", "checl_hostcrc.cpp"]
HEADERS = [os.path.join(CSRC, "checl_internal.h"), os.path.join(ROOT, "include", "checl.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-Wall", f"-I{os.path.join(ROOT, 'include')}"]


def _stale(target: str, deps) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def _build_one(lib: str, obj_dir: str, flags, force: bool, verbose: bool) -> str:
    os.makedirs(obj_dir, exist_ok=True)
    objs, procs = [], []
    for src in SOURCES:  # the three translation units compile in parallel
        path = os.path.join(CSRC, src)
        obj = os.path.join(obj_dir, src + ".o")
        objs.append(obj)
        if force or _stale(obj, [path] + HEADERS):
            cmd = [NVCC, *ARCH, *COMMON, *flags, "-c", path, "-o", obj]
            if verbose and src.endswith(".cu"):
                cmd[1:1] = ["-Xptxas", "-v"]
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            procs.append((cmd, subprocess.Popen(cmd)))
    for cmd, p in procs:
        if p.wait() != 0:
            raise subprocess.CalledProcessError(p.returncode, cmd)
    if force or _stale(lib, objs):
        tmp = lib + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart"])
        os.replace(tmp, lib)
    return lib


def build(force: bool = False, verbose: bool = False, experiments: bool = False) -> str:
    """libchecl.so (the product); with experiments=True also libchecl_exp.so."""
    out = _build_one(LIB, os.path.join(os.path.dirname(LIB), "build_obj" + os.environ.get("CHECL_OBJ_SUFFIX", "")),
                     EXTRA, force, verbose)
    if experiments:
        _build_one(LIB_EXP, os.path.join(PKG, "build_obj_exp"), ["-DCHECL_EXPERIMENTS", *EXTRA], force, verbose)
    return out


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, experiments="--exp" in sys.argv))
