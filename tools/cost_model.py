"""Migration cost model, Eq. (1) (L42-L44 §IV-C, Fig. 8): Tm = alpha*M + Tr + beta.

Measures the process-migration time of this library for checkpoint sizes M on one
B200 box along two routes and fits alpha and beta (Tr = 0: there are no programs to
recompile in a buffer snapshot):
  file   : checkpoint (pinned host image) + write the image file + read it back +
           restore — the paper's route (checkpoint file on one node, restart on another);
  nvlink : checl_migrate (device image, verify+scatter on the destination).
The fit uses every other size; the held-out sizes are predicted (Fig. 8's
measured-vs-predicted comparison). Prints one JSON object.

    python tools/cost_model.py [--dir /dev/shm] [--reps 3]
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402


def fit(ms, ts):
    A = np.vstack([np.array(ms, float), np.ones(len(ms))]).T
    (alpha, beta), *_ = np.linalg.lstsq(A, np.array(ts, float), rcond=None)
    return float(alpha), float(beta)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dir", default="/dev/shm")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--sizes-mib", default="3,16,48,128,256,464,768,1024,2048,4096")
    a = ap.parse_args()
    dev = 0
    torch.cuda.set_device(dev)
    rows = []
    for mib in [int(x) for x in a.sizes_mib.split(",")]:
        # a set shaped like the SDK mix: a few large buffers and small ones
        total = mib << 20
        sizes = [total // 2, total // 4, total // 8, total - total // 2 - total // 4 - total // 8 - 20, 20]
        ts = [torch.empty(s, dtype=torch.uint8, device=dev) for s in sizes]
        for i, t in enumerate(ts):
            checl.debug_fill(t, 77, i)
        torch.cuda.synchronize()
        ctx = checl.Context()
        for t in ts:
            ctx.register(t)
        path = os.path.join(a.dir, f"checl_cost_{os.getpid()}.img")
        img = ctx.checkpoint(dev, epoch=0)  # warm: pinned image + staging
        ctx.restore(img, dev)
        ctx.migrate(dev, dev)
        file_t, mig_t, parts = [], [], []
        for _ in range(a.reps):
            t0 = time.perf_counter()
            ctx.checkpoint(dev, epoch=1, into=img)
            t1 = time.perf_counter()
            img.write(path, direct=True)
            t2 = time.perf_counter()
            back = checl.Image.read(path)
            t3 = time.perf_counter()
            ctx.restore(back, dev)
            t4 = time.perf_counter()
            back.free()
            file_t.append(t4 - t0)
            parts.append((t1 - t0, t2 - t1, t3 - t2, t4 - t3))
            t5 = time.perf_counter()
            ctx.migrate(dev, dev)
            mig_t.append(time.perf_counter() - t5)
        M = img.info()["image_bytes"]
        os.unlink(path)
        img.free()
        ctx.close()
        del ts
        torch.cuda.empty_cache()
        med = lambda xs: statistics.median(xs)  # noqa: E731
        p = [med([x[i] for x in parts]) for i in range(4)]
        rows.append({"M_bytes": M, "file_s": med(file_t), "nvlink_s": med(mig_t), "checkpoint_s": p[0], "write_s": p[1],
                     "read_s": p[2], "restore_s": p[3], "write_GBs": M / p[1] / 1e9, "read_GBs": M / p[2] / 1e9})
    out = {"equation": "Tm = alpha*M + Tr + beta (PAPER.md Eq. 1), Tr = 0", "dir": a.dir, "rows": rows, "routes": {}}
    for route in ("file", "nvlink"):
        ms = [r["M_bytes"] for r in rows]
        ts = [r[f"{route}_s"] for r in rows]
        fit_i = list(range(0, len(rows), 2))
        hold = [i for i in range(len(rows)) if i not in fit_i]
        alpha, beta = fit([ms[i] for i in fit_i], [ts[i] for i in fit_i])
        pred = [alpha * m + beta for m in ms]
        err = [abs(pred[i] - ts[i]) / ts[i] for i in hold]
        ss_res = sum((pred[i] - ts[i]) ** 2 for i in range(len(ms)))
        ss_tot = sum((t - statistics.mean(ts)) ** 2 for t in ts)
        out["routes"][route] = {"alpha_s_per_GB": alpha * 1e9, "effective_GBs": 1 / alpha / 1e9 if alpha > 0 else None,
                                "beta_s": beta, "r2": 1 - ss_res / ss_tot if ss_tot else None,
                                "heldout_rel_err_max": max(err) if err else None,
                                "heldout_rel_err_mean": statistics.mean(err) if err else None,
                                "predicted_s": pred, "measured_s": ts}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
