"""Builds libchecl.so in-tree (nvcc, sm_100a only).

    python -m paper_conf_ipps_takizawakskk11_b200.build [--force]
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.environ.get("CHECL_LIB_OUT", os.path.join(PKG, "libchecl.so"))
OBJ = os.path.join(os.path.dirname(LIB), "build_obj" + os.environ.get("CHECL_OBJ_SUFFIX", ""))
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


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(OBJ, exist_ok=True)
    objs = []
    for src in SOURCES:
        path = os.path.join(CSRC, src)
        obj = os.path.join(OBJ, src + ".o")
        objs.append(obj)
        if force or _stale(obj, [path] + HEADERS):
            cmd = [NVCC, *ARCH, *COMMON, *EXTRA, "-c", path, "-o", obj]
            if verbose and src.endswith(".cu"):
                cmd[1:1] = ["-Xptxas", "-v"]
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            subprocess.check_call(cmd)
    if force or _stale(LIB, objs):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart"])
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
