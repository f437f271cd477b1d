"""Migration cost model, Eq. (1) (L42-L44 §IV-C, Fig. 8): Tm = alpha*M + Tr + beta.

Measures process-migration time of this library for checkpoint sizes M on one B200
box along the routes below, fits alpha and beta on a size sweep (Tr = 0: a buffer
snapshot recompiles nothing; reading 24), and reports predicted vs measured
Tm for the sweep's held-out sizes and for the §8(d) configurations C1-C5 (Fig. 8
compares measured and predicted migration time per benchmark):

  file         the paper's route (a checkpoint file written on one node, read and
               restarted on another): checkpoint into a pinned host image, write the
               file with O_DIRECT and fsync, evict it from the page cache
               (posix_fadvise DONTNEED, plus /proc/sys/vm/drop_caches when writable),
               read it back with O_DIRECT, restore;
  hbm_same_gpu checl_migrate(i, i): K1 into an HBM image and K2 from it on the same
               GPU (no link crossed; what a one-GPU box can measure);
  nvlink       checl_migrate(0, 1) when the box has two GPUs (K2 reads GPU 0's HBM
               over NVLink peer access).

Every point is repeated --reps times (median, min, max reported). Prints one JSON
object.

    python tools/cost_model.py [--dir DIR] [--reps 5] [--configs C1,C2,C3,C5]
"""
import argparse
import json
import os
import statistics
import sys
import time

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(HERE))
sys.path.insert(0, HERE)
import torch  # noqa: E402

import eq1  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_takizawakskk11_b200 import checl  # noqa: E402


def evict(path: str) -> bool:
    """Drops the file's pages from the page cache; True if the global drop ran too."""
    fd = os.open(path, os.O_RDONLY)
    try:
        os.fsync(fd)
        os.posix_fadvise(fd, 0, 0, os.POSIX_FADV_DONTNEED)
    finally:
        os.close(fd)
    try:
        with open("/proc/sys/vm/drop_caches", "w") as f:
            f.write("1\n")
        return True
    except OSError:
        return False


def measure(sizes, reps: int, directory: str, dev: int):
    """One registry of `sizes`; per route the list of `reps` times (s) and the image size."""
    ts = [torch.empty(s, dtype=torch.uint8, device=dev) for s in sizes]
    for i, t in enumerate(ts):
        checl.debug_fill(t, 77, i)
    torch.cuda.synchronize()
    ctx = checl.Context()
    for t in ts:
        ctx.register(t)
    path = os.path.join(directory, f"checl_cost_{os.getpid()}.img")
    img = ctx.checkpoint(dev, epoch=0)  # warm: pinned image, staging, plan
    ctx.restore(img, dev)
    ctx.migrate(dev, dev)
    two = torch.cuda.device_count() > 1
    out = {"file": [], "hbm_same_gpu": [], "nvlink": [], "parts": [], "dropped_caches": False}
    for _ in range(reps):
        t0 = time.perf_counter()
        ctx.checkpoint(dev, epoch=1, into=img)
        t1 = time.perf_counter()
        img.write(path, direct=True, sync=True)
        t2 = time.perf_counter()
        out["dropped_caches"] = evict(path)
        t3 = time.perf_counter()
        back = checl.Image.read(path, direct=True)
        t4 = time.perf_counter()
        ctx.restore(back, dev)
        t5 = time.perf_counter()
        back.free()
        out["file"].append((t2 - t0) + (t5 - t3))  # (the eviction is not migration work)
        out["parts"].append((t1 - t0, t2 - t1, t4 - t3, t5 - t4))
        t6 = time.perf_counter()
        ctx.migrate(dev, dev)
        out["hbm_same_gpu"].append(time.perf_counter() - t6)
        if two:
            ctx.migrate(dev, 1)  # warm the peer path on the first rep
            t7 = time.perf_counter()
            ctx.migrate(1, dev)
            out["nvlink"].append(time.perf_counter() - t7)
    out["M_bytes"] = img.info()["image_bytes"]
    os.unlink(path)
    img.free()
    ctx.close()
    del ts
    torch.cuda.empty_cache()
    return out


def summarise(samples):
    return {"median_s": statistics.median(samples), "min_s": min(samples), "max_s": max(samples), "n": len(samples)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dir", default=os.getcwd(), help="directory on the file system to measure (a real disk)")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--sizes-mib", default="3,16,48,128,256,464,768,1024,2048,4096")
    ap.add_argument("--configs", default="C1,C2,C3,C5")
    a = ap.parse_args()
    dev = 0
    torch.cuda.set_device(dev)
    rows = []
    for mib in [int(x) for x in a.sizes_mib.split(",")]:
        # a set shaped like the SDK mix: a few large buffers and small ones
        total = mib << 20
        sizes = [total // 2, total // 4, total // 8, total - total // 2 - total // 4 - total // 8 - 20, 20]
        r = measure(sizes, a.reps, a.dir, dev)
        p = [statistics.median([x[i] for x in r["parts"]]) for i in range(4)]
        rows.append({"M_bytes": r["M_bytes"], **{k: summarise(r[k]) for k in ("file", "hbm_same_gpu", "nvlink") if r[k]},
                     "checkpoint_s": p[0], "write_s": p[1], "read_s": p[2], "restore_s": p[3],
                     "write_GBs": r["M_bytes"] / p[1] / 1e9, "read_GBs": r["M_bytes"] / p[2] / 1e9,
                     "dropped_caches": r["dropped_caches"]})
    cfg_meas = {}
    for name in [c for c in a.configs.split(",") if c]:
        w = synth.CONFIGS[name]()
        r = measure([b.size for b in w.buffers], a.reps, a.dir, dev)
        cfg_meas[name] = {"workload": w.name, "M_bytes": r["M_bytes"],
                          **{k: summarise(r[k]) for k in ("file", "hbm_same_gpu", "nvlink") if r[k]}}
    out = {"equation": "Tm = alpha*M + Tr + beta (PAPER.md Eq. 1), Tr = 0", "dir": a.dir, "reps": a.reps,
           "rows": rows, "routes": {}}
    fit_i = list(range(0, len(rows), 2))  # every other size; the rest are predicted
    for route in ("file", "hbm_same_gpu", "nvlink"):
        if not all(route in r for r in rows):
            continue
        ms = [r["M_bytes"] for r in rows]
        ts = [r[route]["median_s"] for r in rows]
        res = eq1.evaluate(ms, ts, fit_i)
        alpha, beta = res["alpha_s_per_GB"] / 1e9, res["beta_s"]
        res["configs"] = eq1.predict_configs(alpha, beta, {
            k: {"M_bytes": v["M_bytes"], "measured_s": v[route]["median_s"]} for k, v in cfg_meas.items() if route in v})
        out["routes"][route] = res
    print(json.dumps(out))


if __name__ == "__main__":
    main()
