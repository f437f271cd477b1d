import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from oracle import oracle as O
from tests.gpu_util import make_set, oracle_entries, bound_bytes
from paper_conf_ipps_takizawakskk11_b200 import checl
sizes = [1 << 20, 0, 65536 * 3 + 17, 4097, 1, 300007, 65535, 65537, 2 << 20]
ctx = checl.Context()
ds = make_set(ctx, sizes, seed=21, offsets=[0, 0, 1, 4, 0, 8, 3, 0, 0])
want = O.checkpoint(oracle_entries(ds), device=0, epoch=3)
img = ctx.checkpoint(0, epoch=3)
print("eq", np.array_equal(img.view(), want))
