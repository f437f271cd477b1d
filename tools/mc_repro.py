"""Repro/diagnostic for the multicast table prologue (CHECL_TABLE_MC=1): the forced
kernel-4 registry of tests/test_gpu_kernels.py, reporting where images differ."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
from oracle import oracle as O  # noqa: E402
from tests.gpu_util import make_set, oracle_entries  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402

sizes = [1 << 20, 0, 65536 * 3 + 17, 4097, 1, 300007, 65535, 65537, 2 << 20]
for slot in (None, 196608):
    for rep in range(3):
        ctx = checl.Context()
        if slot:
            ctx.set_staging(slot, 2)
        ds = make_set(ctx, sizes, seed=21, offsets=[0, 0, 1, 4, 0, 8, 3, 0, 0])
        want = O.checkpoint(oracle_entries(ds), device=0, epoch=3)
        img = ctx.checkpoint(0, epoch=3)
        got = img.view()
        hd = img.header()
        bad = np.nonzero(got != want)[0]
        if bad.size == 0:
            print(f"slot {slot} rep {rep}: ok")
        else:
            crc_lo, pay = hd["crc_off"], hd["payload_off"]
            in_crc = bad[(bad >= crc_lo) & (bad < pay)]
            in_pay = bad[bad >= pay]
            chunks_crc = sorted(set(((in_crc - crc_lo) // 4).tolist()))
            chunks_pay = sorted(set(((in_pay - pay) // 65536).tolist()))
            print(f"slot {slot} rep {rep}: {bad.size} bytes differ; crc entries {chunks_crc[:20]} "
                  f"payload 64K-blocks {chunks_pay[:20]} meta {int((bad < crc_lo).sum())}")
            for blk in chunks_pay[:4]:
                lo = pay + blk * 65536
                g, w_ = got[lo:lo + 65536], want[lo:lo + 65536]
                rounds = "".join("x" if (g[r * 4096:(r + 1) * 4096] != w_[r * 4096:(r + 1) * 4096]).any() else "."
                                 for r in range(16))
                zeros = "".join("0" if not g[r * 4096:(r + 1) * 4096].any() else "-" for r in range(16))
                print(f"   block {blk}: rounds differ {rounds}  all-zero {zeros}")
        ctx.close()
