"""Benchmark of the CheCL snapshot hot path (checkpoint -> coordinate -> restore).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--kind random]
    python bench.py --impl reference ...     # the CPU oracle on the same workload

One step = one pass of every SURVEY.md §8(a) row over the workload's buffers:
a1 sync, a2 plan, a3 pack+CRC (K1), a4 drain, a5 finalize, a6 coordination
all-reduce (N > 1), r1 validate, r2 re-create, r3 fill, r4 verify+scatter (K2),
r5 rebind. `value` keeps the image resident in HBM (a4/r3 are HBM-resident, the
path `checl_migrate` uses); `e2e` is the same step through the C ABI with the
image in pinned HOST memory (PCIe D2H drain + H2D fill inside the timed region).
Metric: payload GB/s of checkpoint + restore = bytes / (t_checkpoint + t_restore),
summed over ranks, timed with CUDA events, max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "checkpoint & restore GB/s per GPU and box (1/2/4/8), % of HBM/PCIe roofline"
L2_BYTES = 126 * 2**20


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    # default: configs[2] (C3, 10 000 odd buffers, 5.26 GB), the largest configuration that
    # runs on one GPU with its buffers, image and restored copy all resident (C4's 64 GiB
    # needs restart mode); C2 and C4 ride along as extra fields at N = 1
    ap.add_argument("--config", default="C3", choices=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--no-extras", action="store_true", help="skip the C2 / C4 extra fields (N = 1)")
    ap.add_argument("--extra-steps", type=int, default=10)
    ap.add_argument("--kind", default="random", choices=["random", "float", "zeros"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--c4-scale", type=float, default=1.0)
    ap.add_argument("--restart", action="store_true",
                    help="every step releases all handles between checkpoint and restore (the restarted process "
                         "holds only the image; automatic when buffers + image + restored copy exceed HBM)")
    ap.add_argument("--c5-large", action="store_true", help="C5 with 16 x 1 GiB instead of the C2 set")
    ap.add_argument("--c5-route", default="peer", choices=["peer", "copy"],
                    help="C5 A/B: K2 reads the source GPU's HBM over NVLink (peer), or the copy engine moves the "
                         "image first and K2 runs locally (copy)")
    ap.add_argument("--mode", default="snapshot", choices=["snapshot", "incremental"],
                    help="incremental: checl_checkpoint_incremental with --dirty of the chunks rewritten per step")
    ap.add_argument("--dirty", type=float, default=0.1)
    ap.add_argument("--rule", default="bytes", choices=["bytes", "crc"],
                    help="incremental dirty rule: bytes (exact, default) or crc (fast option)")
    return ap.parse_args()


def workload(cfg: str, rank: int, c4_scale: float):
    import synth
    if cfg == "C4":
        return synth.c4_md_rank(rank, c4_scale)
    w = synth.CONFIGS[cfg]()
    w.seed += 1000 * rank
    return w


def init_dist(dist, torch, dev):
    """One process per GPU over NCCL. CHECL_BENCH_DIST_BACKEND=gloo is for exercising
    the multi-rank code path with several ranks on one GPU (timings meaningless)."""
    backend = os.environ.get("CHECL_BENCH_DIST_BACKEND", "nccl")
    if backend == "nccl":
        dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
    else:
        dist.init_process_group(backend)


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == 7:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[3 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def pcie_probe(dev: int, snap=None, nbytes: int = 256 << 20):
    """Pinned D2H / H2D copy bandwidth (torch plumbing, untimed region): the PCIe
    roofline. With several ranks every rank probes at the same time (barrier first), so
    the denominator is the all-ranks-concurrent bandwidth the e2e leg also sees; the
    per-rank figures and their sum over ranks (the box) are reported."""
    import torch
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    out = {}
    s = torch.cuda.Stream(dev)
    for name, fn in (("d2h", lambda: h.copy_(d, non_blocking=True)), ("h2d", lambda: d.copy_(h, non_blocking=True))):
        with torch.cuda.stream(s):
            fn()
            fn()
        s.synchronize()
        if snap is not None:
            snap.barrier()
        with torch.cuda.stream(s):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(5):
                fn()
            e1.record(s)
        e1.synchronize()
        out[name] = nbytes * 5 / (e0.elapsed_time(e1) * 1e-3) / 1e9
    del h, d
    if snap is not None and snap.world > 1:
        import torch.distributed as dist
        out["box_d2h"] = snap.over_ranks(out["d2h"], dist.ReduceOp.SUM)
        out["box_h2d"] = snap.over_ranks(out["h2d"], dist.ReduceOp.SUM)
        out["concurrent_ranks"] = snap.world
    return out


def cpu_baseline(w, max_seconds: float = 20.0):
    """The oracle (oracle/, as it stands) on the same workload: checkpoint + restore."""
    import numpy as np
    import synth
    from oracle import oracle as O
    total = w.total_bytes
    # bounded sample: whole buffers in order until ~1.5 GB (C2 fits whole)
    picked, acc = [], 0
    for b in w.buffers:
        if picked and acc + b.size > 1_500_000_000:
            break
        picked.append(b)
        acc += b.size
    ents = [O.Entry(i + 1, synth.fill_bytes(b.size, w.seed, b.stream), b.flags) for i, b in enumerate(picked)]
    times = []
    t_start = time.perf_counter()
    while True:
        t0 = time.perf_counter()
        img = O.checkpoint(ents, device=0, epoch=1)
        st, rep, back = O.restore(img)
        t = time.perf_counter() - t0
        assert st == 0
        times.append(t)
        del img, back
        if time.perf_counter() - t_start > max_seconds or len(times) >= 3:
            break
    t = statistics.median(times)
    sample = (f"{len(picked)}/{len(w.buffers)} buffers of {w.name} ({acc} of {total} B), "
              f"oracle checkpoint+restore, median of {len(times)}")
    return {"value": acc / t / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": sample,
            "ms_per_roundtrip": t * 1e3, "cpu_model": cpu_model()}


def cpu_model() -> str:
    """The host CPU's model name (/proc/cpuinfo), recorded beside the oracle's timing."""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def run_reference(a):
    """--impl reference: the oracle, as it stands, on the host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import numpy as np
    import synth
    from oracle import oracle as O
    w = workload(a.config, 0, a.c4_scale)
    picked, acc = [], 0
    budget = 600_000_000  # bounded sample per step so K steps end within minutes
    for b in w.buffers:
        if picked and acc + b.size > budget:
            break
        picked.append(b)
        acc += b.size
    ents = [O.Entry(i + 1, synth.fill_bytes(b.size, w.seed, b.stream), b.flags) for i, b in enumerate(picked)]
    for _ in range(a.warmup):
        O.restore(O.checkpoint(ents, 0, 1))
    t0 = time.perf_counter()
    for _ in range(a.steps):
        img = O.checkpoint(ents, 0, 1)
        st, _, _ = O.restore(img)
        assert st == 0
    dt = time.perf_counter() - t0
    value = acc * a.steps / dt / 1e9
    sample = f"{len(picked)}/{len(w.buffers)} buffers of {w.name}, {acc} B per step (oracle pack+CRC+restore, 1 thread)"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": a.gpus, "steps": a.steps,
        "warmup": a.warmup, "ms_per_step": dt / a.steps * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": w.name, "payload_bytes_per_gpu": w.total_bytes, "n_buffers": len(w.buffers)},
        "cpu_baseline": {"value": value, "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": sample,
                         "cpu_model": cpu_model()},
        "e2e": {"value": value, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


def run_migration(a):
    """configs[4] (C5): every rank migrates its buffers GPU i -> GPU (i+1) mod n
    (m1-m3: K1 into an HBM image on i, K2 on the destination reading it over NVLink
    peer memory). With one GPU the destination is the source (no NVLink crossing)."""
    import torch
    import torch.distributed as dist
    import synth
    from paper_conf_ipps_takizawakskk11_b200 import checl

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    ndev = torch.cuda.device_count()
    dev = int(os.environ.get("LOCAL_RANK", "0")) % max(ndev, 1)
    torch.cuda.set_device(dev)
    if world > 1:
        init_dist(dist, torch, dev)
    nvlink = nvlink_probe(dev, ndev, world, dist)
    w = synth.c5_migration(large=a.c5_large)
    tensors = [torch.empty(b.size, dtype=torch.uint8, device=dev) for b in w.buffers]
    for t, b in zip(tensors, w.buffers):
        checl.debug_fill(t, w.seed, b.stream)
    torch.cuda.synchronize()
    ctx = checl.Context()
    handles = [ctx.register(t) for t in tensors]
    S = w.total_bytes
    cur = dev
    def target(c):
        return (c + 1) % ndev if world > 1 else c

    for _ in range(a.warmup):
        nxt = target(cur)
        ctx.migrate(cur, nxt)
        cur = nxt
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    timings = []
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.steps):
        nxt = target(cur)
        ctx.migrate(cur, nxt)
        timings.append(ctx.last_timing())
        cur = nxt
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1)
    n_diff = 0
    for h, t in zip(handles, tensors):
        ptr, nb, d = ctx.translate(h)
        if d == dev:
            n_diff += checl.debug_compare(dev, ptr, t.data_ptr(), nb)
        elif nb:  # the buffers now live on another GPU: bring them back (torch peer copy) to compare
            n_diff += int(not torch.equal(ctx.tensor(h).to(dev), t))
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    if rank == 0:
        kern = statistics.mean(t["kernel_ms"] for t in timings)
        crosses = world > 1 and ndev > 1
        route = ("same GPU (1 device)" if not crosses else
                 "copy engine (cudaMemcpyPeerAsync) + local K2" if os.environ.get("CHECL_FORCE_NO_PEER")
                 else "K2 reads the peer's HBM over NVLink")
        per_gpu = S / (ms / a.steps * 1e-3) / 1e9
        print(json.dumps({
            "metric": "in-box migration GB/s (checl_migrate, GPU i -> GPU (i+1) mod n)", "value": S * world * a.steps / (ms * 1e-3) / 1e9,
            "unit": "GB/s", "n_gpus": world, "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms / a.steps,
            "config": {"workload": w.name, "payload_bytes_per_gpu": S, "n_buffers": len(w.buffers), "route": route},
            "kernel_ms_per_step": kern, "kernels_2S_GBs": 4 * S / (kern * 1e-3) / 1e9,
            "nvlink_roofline": (dict(nvlink, achieved_GBs_per_gpu=per_gpu,
                                     frac=per_gpu / nvlink["peer_copy_GBs"]) if nvlink.get("peer_copy_GBs") else nvlink),
            "verified": n_diff == 0, "last_timing": timings[-1]}))
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


def nvlink_probe(dev: int, ndev: int, world: int, dist) -> dict:
    """The NVLink roofline of migration: cudaMemcpyPeerAsync (torch's
    peer copy) of 1 GiB from this rank's GPU to the next one, all ranks at once (the
    i -> (i+1) mod n pattern of C5). None on a one-GPU box."""
    import torch
    if world == 1 or ndev < 2:
        return {"peer_copy_GBs": None, "note": "one GPU: no NVLink crossing to measure"}
    nxt = (dev + 1) % ndev
    n = 1 << 30
    src = torch.empty(n, dtype=torch.uint8, device=dev)
    dst = torch.empty(n, dtype=torch.uint8, device=nxt)
    s = torch.cuda.Stream(dev)
    with torch.cuda.stream(s):
        dst.copy_(src, non_blocking=True)
    s.synchronize()
    dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s)
        for _ in range(5):
            dst.copy_(src, non_blocking=True)
        e1.record(s)
    e1.synchronize()
    del src, dst
    return {"peer_copy_GBs": 5 * n / (e0.elapsed_time(e1) * 1e-3) / 1e9, "pattern": "GPU i -> GPU (i+1) mod n, all ranks"}


def run_incremental(a):
    """incremental checkpoint (PAPER.md L45 future work). Between
    steps the "application" rewrites one byte in a fraction `--dirty` of the
    workload's chunks (untimed); each timed step is checl_checkpoint_incremental on
    the previous image (pinned host image, PCIe drain of the changed chunks only).
    Reported next to a full checkpoint of the same workload and a chain restore."""
    import numpy as np
    import torch
    from paper_conf_ipps_takizawakskk11_b200 import checl

    dev = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(dev)
    w = workload(a.config, 0, a.c4_scale)
    tensors = [torch.empty(b.size, dtype=torch.uint8, device=dev) for b in w.buffers]
    for t, b in zip(tensors, w.buffers):
        checl.debug_fill(t, w.seed, b.stream)
    torch.cuda.synchronize()
    ctx = checl.Context()
    for t, b in zip(tensors, w.buffers):
        ctx.register(t, b.flags)
    S = w.total_bytes
    # chunk start positions (buffer, offset) for the mutation
    starts = [(i, j * 65536) for i, b in enumerate(w.buffers) for j in range((b.size + 65535) // 65536)]
    rng = np.random.default_rng(5)
    k = max(1, int(len(starts) * a.dirty))

    def mutate():
        pick = rng.choice(len(starts), size=k, replace=False)
        by_buf = {}
        for c in pick:
            i, o = starts[c]
            by_buf.setdefault(i, []).append(o + int(rng.integers(0, min(65536, w.buffers[i].size - o))))
        for i, offs in by_buf.items():
            idx = torch.tensor(offs, dtype=torch.int64, device=dev)
            tensors[i][idx] ^= 0x5A
        torch.cuda.synchronize()

    cur = torch.cuda.current_stream(dev)
    rule = checl.DIRTY_BYTES if a.rule == "bytes" else checl.DIRTY_CRC

    def timed(fn):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(cur)
        r = fn()
        e1.record(cur)
        e1.synchronize()
        return e0.elapsed_time(e1), r

    full = ctx.checkpoint(dev, epoch=0)
    full_ms = []
    for i in range(a.warmup + a.steps):
        ms, _ = timed(lambda: ctx.checkpoint(dev, epoch=0, into=full))
        if i >= a.warmup:
            full_ms.append(ms)
    base = full

    def advance(d):
        # the previous delta has served as base: free it (its pinned buffer goes back to
        # the library's pool, as an application would after writing it out)
        nonlocal base
        if base is not full:
            base.free()
        base = d

    for i in range(a.warmup):
        mutate()
        advance(ctx.checkpoint_incremental(dev, base, epoch=i + 1, rule=rule))
    ms_steps, drained, present, tms = [], [], [], []
    with ClockSampler(dev) as clk:
        for i in range(a.steps):
            mutate()
            ms, d = timed(lambda: ctx.checkpoint_incremental(dev, base, epoch=a.warmup + i + 1, rule=rule))
            h = d.header()
            ms_steps.append(ms)
            drained.append(h["payload_bytes"])
            present.append(h["n_present"])
            tms.append(ctx.last_timing())
            advance(d)
    # chain restore of [full, last delta] is not linked (intermediate deltas freed):
    # restore [merge(full@now), ...] instead: take a fresh full and one delta
    f2 = ctx.checkpoint(dev, epoch=100)
    mutate()
    d2 = ctx.checkpoint_incremental(dev, f2, epoch=101, rule=rule)
    # the first two calls allocate the re-created segments (5.35 GB through cudaMalloc for
    # C3: ~1 s); from the third on they come from the spares of the previous commit
    chain = [timed(lambda: ctx.restore_chain([f2, d2], dev)) for _ in range(5)]
    rs_ms, rep = statistics.median(c[0] for c in chain[2:]), chain[-1][1]
    n_diff = 0
    for h, t in zip(range(1, len(tensors) + 1), tensors):
        ptr, nb, _ = ctx.translate(h)
        n_diff += checl.debug_compare(dev, ptr, t.data_ptr(), nb) if nb else 0
    t_inc = statistics.median(ms_steps)
    t_full = statistics.median(full_ms)
    crc_ms = statistics.mean(t["kernel_ms"] for t in tms)
    pk = peaks()
    hbm = pk.get("hbm_gbs") or 6650.0
    print(json.dumps({
        "metric": "incremental checkpoint GB/s (logical payload / time), pinned host image",
        "value": S / (t_inc * 1e-3) / 1e9, "unit": "GB/s", "n_gpus": 1, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": t_inc, "ms_per_step_all": ms_steps, "higher_is_better": True, "dtype": "u8", "data": "synthetic",
        "config": {"workload": w.name, "payload_bytes_per_gpu": S, "n_chunks": len(starts),
                   "dirty_fraction": a.dirty, "chunks_rewritten_per_step": k, "dirty_rule": a.rule},
        "full_checkpoint_ms": t_full, "speedup_vs_full": t_full / t_inc,
        "drained_bytes_per_step": statistics.mean(drained), "present_chunks_per_step": statistics.mean(present),
        "kernel_ms_per_step": crc_ms,
        "dirty_pass": ({"bytes_read": 2 * S, "note": "diff_kernel reads S (buffers) + S (shadow), writes the "
                        "changed rounds; gather + CRC of the present spans only"} if a.rule == "bytes" else
                       {"bytes_read": S, "note": "kOpCrc reads S; gather reads + writes only the present spans"}),
        "last_timing": tms[-1], "chain_restore_ms": rs_ms, "chain_restore_ms_all": [c[0] for c in chain], "chain_restore_GBs": S / (rs_ms * 1e-3) / 1e9,
        "verified": n_diff == 0 and rep.n_bad_chunks == 0, "clocks": clk.summary(), "hbm_peak": hbm}))
    ctx.close()


def restart_samples_bad(ctx, handles, w, kind: str, per_buffer: int = 8) -> int:
    """Restart mode: sampled 64 KiB chunks (random ones + each buffer's last) of the
    restored buffers vs the synth generator's bytes; the number that differ."""
    import numpy as np
    import synth
    rng = np.random.default_rng(w.seed)
    bad = 0
    for h, b in zip(handles, w.buffers):
        nch = (b.size + 65535) // 65536
        if nch == 0:
            continue
        t = ctx.tensor(h)
        for k in [int(x) for x in rng.integers(0, nch, per_buffer)] + [nch - 1]:
            lo, n = k * 65536, min(65536, b.size - k * 65536)
            bad += int(not np.array_equal(t[lo:lo + n].cpu().numpy(), synth.fill_slice(lo, n, w.seed, b.stream, kind)))
    return bad


def meminfo_available() -> int:
    """MemAvailable of the host (bytes), or 0 when unknown."""
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("MemAvailable:"):
                return int(line.split()[1]) * 1024
    except OSError:
        pass
    return 0


def copy_same_size(torch, dev: int, S: int, achieved: float) -> dict:
    """Context for the roofline: torch's own device copy (b.copy_(a), the op the
    MEASURED_PEAKS.json copy peak is taken with, at 2 GiB) of the workload's payload
    size, CUDA events around each copy, median of 5 after one warm-up. Not the peak:
    a copy's rate depends on its size."""
    free, _ = torch.cuda.mem_get_info(dev)
    n = min(S, (free - (1 << 30)) // 2 // (1 << 20) * (1 << 20))  # C4 in restart mode: what fits
    if n < (256 << 20):
        return {"GBs": None, "reason": f"{free} B of free HBM"}
    try:
        a = torch.empty(n, dtype=torch.uint8, device=dev)
        b = torch.empty_like(a)
    except torch.cuda.OutOfMemoryError as e:  # context only: never fail the run for it
        torch.cuda.empty_cache()
        return {"GBs": None, "reason": f"allocation failed: {str(e)[:80]}"}
    a.fill_(1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for i in range(6):
        torch.cuda.synchronize(dev)
        e0.record()
        b.copy_(a)
        e1.record()
        torch.cuda.synchronize(dev)
        if i:
            ts.append(e0.elapsed_time(e1))
    del a, b
    torch.cuda.empty_cache()
    ts.sort()
    rate = 2 * n / (ts[len(ts) // 2] * 1e-3) / 1e9
    return {"GBs": rate, "frac": achieved / rate, "bytes": n,
            "how": "torch b.copy_(a) of the payload size (or the largest that fits), median of 5"}


def traffic_entry(cfg: str, kernel: str):
    """ncu --set full DRAM bytes per launch of the dominant kernel (profiles/traffic.json)."""
    tf = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        t = json.load(open(tf)).get(cfg, {})
        return t.get(kernel, t.get("dram_bytes_per_launch")), t.get("source")
    except Exception:
        return None, None


class Snapshot:
    """One workload's checkpoint -> coordinate -> restore loop on
    this rank's GPU: `value` with the image in HBM, `e2e` with a pinned host image."""

    def __init__(self, a, cfg: str, rank: int, world: int, dev: int, dist, c4_scale: float = 1.0,
                 restart: bool = False):
        import torch
        from paper_conf_ipps_takizawakskk11_b200 import checl
        self.a, self.cfg, self.rank, self.world, self.dev, self.dist = a, cfg, rank, world, dev, dist
        self.torch, self.checl = torch, checl
        self.w = workload(cfg, rank, c4_scale)
        self.kind = {"random": checl.FILL_RANDOM, "float": checl.FILL_FLOAT, "zeros": checl.FILL_ZEROS}[a.kind]
        # the application's buffers (user-owned), filled on the device by the synth/ generator
        self.tensors = [torch.empty(b.size, dtype=torch.uint8, device=dev) for b in self.w.buffers]
        for t, b in zip(self.tensors, self.w.buffers):
            checl.debug_fill(t, self.w.seed, b.stream, self.kind)
        torch.cuda.synchronize()
        self.ctx = checl.Context()
        self.handles = [self.ctx.register(t, b.flags) for t, b in zip(self.tensors, self.w.buffers)]
        self.S = self.w.total_bytes
        self.n_chunks = sum((b.size + 65535) // 65536 for b in self.w.buffers)
        # Restart mode (L16 restart steps 2-3: the new process re-creates every object from
        # the image). The application's buffers are dropped after the first checkpoint and
        # every timed step releases all handles before restoring, so HBM holds one image
        # plus one copy of the buffers: C4 at full size (64 GiB x 3 does not fit 179 GiB).
        self.restart = restart or 3 * self.S + (4 << 30) > torch.cuda.get_device_properties(dev).total_memory
        # inputs smaller than L2: every timed step starts from a flushed L2 (a 2x-L2
        # buffer written between steps, outside the timed spans)
        self.flush = torch.empty(2 * L2_BYTES, dtype=torch.uint8, device=dev) if self.S <= L2_BYTES else None

    def over_ranks(self, x: float, op) -> float:
        if self.world == 1:
            return x
        dist, torch = self.dist, self.torch
        t = torch.tensor([x], dtype=torch.float64, device=self.dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(t, op=op)
        return float(t.item())

    def barrier(self):
        if self.world > 1:
            self.dist.barrier()
        self.torch.cuda.synchronize()

    def run(self, img, steps, collect: bool):
        """steps x (checkpoint_into img -> coordinate (a6: the global snapshot's status
        all-reduce with the local checkpoint's real outcome, N > 1) -> restore img);
        returns device ms and, with collect, the library's cumulative per-call timing of
        those steps (checl_stats: kernel spans from its CUDA events, read after the timed
        region)."""
        from paper_conf_ipps_takizawakskk11_b200.coordination import coordinated
        torch, ctx, dev = self.torch, self.ctx, self.dev
        cur = torch.cuda.current_stream(dev)
        total = 0.0
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ctx.reset_stats()
        n_h, S = len(self.handles), self.S
        if self.flush is None:
            e0.record(cur)
        for i in range(steps):
            if self.flush is not None:
                self.flush.fill_(i & 0xFF)
                e0.record(cur)
            if self.world > 1:
                snap = coordinated(lambda: (ctx.checkpoint(dev, epoch=i + 1, into=img), n_h, S), i + 1,
                                   device=dev, keep=img)
                assert snap.committed, "global snapshot aborted"
            else:
                ctx.checkpoint(dev, epoch=i + 1, into=img)
            if self.restart:
                for h in self.handles:
                    ctx.release(h)
            ctx.restore(img, dev, report=False)
            if self.flush is not None:
                e1.record(cur)
                e1.synchronize()
                total += e0.elapsed_time(e1)
        if self.flush is None:
            e1.record(cur)
            e1.synchronize()
            total = e0.elapsed_time(e1)
        if not collect:
            return total, None
        checl = self.checl
        st = (ctx.stats(checl.STATS_CHECKPOINT), ctx.stats(checl.STATS_RESTORE))
        assert st[0]["n_calls"] == steps and st[1]["n_calls"] == steps
        return total, st

    def detail(self, img):
        """One more (untimed) step: the per-phase timing of a checkpoint and a restore."""
        ctx = self.ctx
        ctx.checkpoint(self.dev, epoch=self.a.steps + 1, into=img)
        tc = ctx.last_timing()
        if self.restart:
            for h in self.handles:
                ctx.release(h)
        ctx.restore(img, self.dev, report=False)
        return tc, ctx.last_timing()

    def device_image(self, steps: int, warmup: int, clocks: bool = True) -> dict:
        """value: the image resident in HBM (the checl_migrate path), inputs > L2 or L2 flushed."""
        torch, ctx, dev, S, n_chunks = self.torch, self.ctx, self.dev, self.S, self.n_chunks
        dimg = ctx.checkpoint_device(dev, epoch=0)
        crc0 = None
        if self.restart:
            import numpy as np
            hd = dimg.header()
            crc0 = np.array(dimg.view()[hd["crc_off"]:hd["crc_off"] + 4 * n_chunks])
            for h in self.handles:
                ctx.release(h)
            self.tensors.clear()  # the user's buffers are gone; only the image survives
            torch.cuda.empty_cache()
            ctx.restore(dimg, dev, report=False)
        self.run(dimg, warmup, False)
        self.barrier()
        with ClockSampler(dev) as clk:
            ms, (sck, srs) = self.run(dimg, steps, True)
        self.barrier()
        last_ck, last_rs = self.detail(dimg)
        ms_max = self.over_ranks(ms, self.dist.ReduceOp.MAX if self.world > 1 else None)
        value = self.over_ranks(S * steps, self.dist.ReduceOp.SUM if self.world > 1 else None) / (ms_max * 1e-3) / 1e9
        # correctness of the last restore: every handle's new buffer == the application's bytes
        n_diff = 0
        for h, t in zip(self.handles, self.tensors):
            ptr, nb, d = ctx.translate(h)
            n_diff += self.checl.debug_compare(dev, ptr, t.data_ptr(), nb) if nb else 0
        if self.restart:
            # no original left to compare with: the last image's CRC table must equal the
            # first one's (taken from the application's buffers), and sampled chunks of the
            # restored buffers must equal the synth generator's bytes
            hd = dimg.header()
            n_diff += int(not (dimg.view()[hd["crc_off"]:hd["crc_off"] + 4 * n_chunks] == crc0).all())
            n_diff += restart_samples_bad(ctx, self.handles, self.w, self.a.kind)
        pack_ms = sck["kernel_ms"] / sck["n_calls"]
        verify_ms = srs["kernel_ms"] / srs["n_calls"]
        ck_ms = sck["total_ms"] / sck["n_calls"]
        rs_ms = srs["total_ms"] / srs["n_calls"]
        pk = peaks()
        hbm_peak = pk.get("hbm_gbs")
        peak_src = "MEASURED_PEAKS.json hbm_gbs (measured copy)" if hbm_peak else "fallback 6650 GB/s (B200_PROFILING.md)"
        hbm_peak = hbm_peak or 6650.0
        alg = 2 * S + 4 * n_chunks  # K1: read S + write S + CRC table; K2: read S + write S + read table
        dom_ms, dom_name = (pack_ms, "pack_gather_crc (K1)") if pack_ms >= verify_ms else (verify_ms, "verify_scatter (K2)")
        achieved = alg / (dom_ms * 1e-3) / 1e9
        traffic, tsrc = traffic_entry(self.cfg, "K1" if dom_name.startswith("pack") else "K2")
        dimg.free()
        same_size = copy_same_size(torch, dev, S, achieved)
        return {
            "value": value, "ms_max": ms_max, "ms_per_step": ms_max / steps, "verified": n_diff == 0,
            "gpu_launches": sck["n_kernels"] + srs["n_kernels"], "clocks": clk.summary(),
            "roofline": {"bound": "hbm", "kernel": dom_name, "achieved": achieved, "peak": hbm_peak,
                         "unit": "GB/s", "frac": achieved / hbm_peak, "traffic": traffic, "traffic_source": tsrc,
                         "peak_source": peak_src, "algorithmic_bytes_per_launch": alg,
                         "launches_per_step": {"K1": sck["n_kernels"] / steps, "K2": srs["n_kernels"] / steps},
                         "pack_ms": pack_ms, "verify_ms": verify_ms, "copy_same_size": same_size},
            "phases": {"checkpoint_ms": ck_ms, "restore_ms": rs_ms, "checkpoint_GBs": S / (ck_ms * 1e-3) / 1e9,
                       "restore_GBs": S / (rs_ms * 1e-3) / 1e9,
                       "pack_GBs_2S": 2 * S / (pack_ms * 1e-3) / 1e9, "verify_GBs_2S": 2 * S / (verify_ms * 1e-3) / 1e9,
                       "checkpoint_detail": last_ck, "restore_detail": last_rs},
        }

    def host_image(self, steps: int, warmup: int) -> dict:
        """e2e: the same step through the C ABI with the image in pinned HOST memory
        (PCIe D2H drain and H2D fill inside the timed region)."""
        ctx, dev, S, n_chunks = self.ctx, self.dev, self.S, self.n_chunks
        pcie = pcie_probe(dev, self)
        himg = ctx.checkpoint(dev, epoch=0)
        payload_span = himg.info()["image_bytes"]
        self.run(himg, warmup, False)
        self.barrier()
        ms2, (eck, ers) = self.run(himg, steps, True)
        self.barrier()
        ms2_max = self.over_ranks(ms2, self.dist.ReduceOp.MAX if self.world > 1 else None)
        E = self.over_ranks(S * steps, self.dist.ReduceOp.SUM if self.world > 1 else None) / (ms2_max * 1e-3) / 1e9
        ck2 = eck["total_ms"] / eck["n_calls"]
        rs2 = ers["total_ms"] / ers["n_calls"]
        drain = eck["copy_ms"] / eck["n_calls"]
        fill = ers["copy_ms"] / ers["n_calls"]
        himg.free()
        pay = S  # payload bytes carried each way (+ padding, tables below)
        return {
            "value": E, "unit": "GB/s",
            "h2d_bytes_per_step": payload_span + 20 * n_chunks + 16,  # image payload + CRC table + descriptors + status
            "d2h_bytes_per_step": payload_span + 4 * n_chunks + 16,   # payload + CRC table + status word
            "checkpoint_ms": ck2, "restore_ms": rs2,
            "checkpoint_GBs": pay / (ck2 * 1e-3) / 1e9, "restore_GBs": pay / (rs2 * 1e-3) / 1e9,
            "drain_GBs": pay / (drain * 1e-3) / 1e9, "fill_GBs": pay / (fill * 1e-3) / 1e9,
            "pcie_measured_GBs": pcie,
            "drain_frac_of_pcie": (pay / (drain * 1e-3) / 1e9) / pcie["d2h"],
            "fill_frac_of_pcie": (pay / (fill * 1e-3) / 1e9) / pcie["h2d"],
            "gpu_launches": eck["n_kernels"] + ers["n_kernels"],
            "image": "pinned host memory (cudaHostAlloc), reused across steps",
        }

    def close(self):
        for h in self.handles:
            try:
                self.ctx.release(h)
            except Exception:
                pass
        self.ctx.close()
        self.tensors.clear()
        self.flush = None
        self.torch.cuda.synchronize()
        self.torch.cuda.empty_cache()


def host_ram_check(image_bytes: int, local_world: int):
    """Pinned host RAM the e2e leg needs on this box (every local rank pins one image)
    against MemAvailable: (fits, needed, available)."""
    need = image_bytes * local_world
    avail = meminfo_available()
    return (avail == 0 or need <= 0.7 * avail), need, avail


def main():
    a = parse()
    if a.mode == "incremental":
        run_incremental(a)
        return
    if a.impl == "reference":
        run_reference(a)
        return
    if a.config == "C5":
        if a.c5_route == "copy":
            os.environ["CHECL_FORCE_NO_PEER"] = "1"  # read once by libchecl (before its first migrate)
        run_migration(a)
        return
    import torch
    import torch.distributed as dist

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", str(world)))
    dev = local % max(torch.cuda.device_count(), 1)  # (== local on a box with a GPU per rank)
    torch.cuda.set_device(dev)
    if world > 1:
        init_dist(dist, torch, dev)

    snap = Snapshot(a, a.config, rank, world, dev, dist, a.c4_scale, a.restart)
    w, S, n_chunks = snap.w, snap.S, snap.n_chunks
    main_res = snap.device_image(a.steps, a.warmup)

    e2e = None
    if not a.no_e2e:
        fits, need, avail = host_ram_check(S + 4 * n_chunks + 48 * len(w.buffers) + (1 << 20), local_world)
        if fits:
            e2e = snap.host_image(a.steps, a.warmup)
        elif w.name.startswith("C4"):
            # scale the MD rank down until every local rank's pinned image fits 70 % of RAM
            scale = max(0.01, min(1.0, 0.7 * avail / local_world / (S * 1.01)))
            snap.close()
            small = Snapshot(a, "C4", rank, world, dev, dist, a.c4_scale * scale)
            e2e = small.host_image(a.steps, a.warmup)
            e2e["scaled_down"] = {"workload": small.w.name, "payload_bytes_per_gpu": small.S, "scale": scale,
                                  "reason": f"{need / 2**30:.0f} GiB of pinned host RAM needed for {local_world} "
                                            f"rank(s), {avail / 2**30:.0f} GiB available"}
            small.close()
        else:
            e2e = {"value": None, "skipped": f"needs {need / 2**30:.1f} GiB pinned host RAM, {avail / 2**30:.1f} available"}
    snap.close()

    # the other single-GPU configs of §8(d) as extra fields (N = 1 only): C2 (configs[1])
    # and C4 at full size in restart mode (configs[3] on one B200)
    extras = {}
    if world == 1 and not a.no_extras:
        for cfg in [c for c in ("C2", "C4") if c != a.config]:
            try:
                ex = Snapshot(a, cfg, rank, world, dev, dist)
                r = ex.device_image(a.extra_steps, a.warmup)
                item = {"workload": ex.w.name, "payload_bytes_per_gpu": ex.S, "n_buffers": len(ex.w.buffers),
                        "restart": ex.restart, "value": r["value"], "unit": "GB/s", "ms_per_step": r["ms_per_step"],
                        "steps": a.extra_steps, "verified": r["verified"], "roofline": r["roofline"],
                        "clocks": r["clocks"], "phases": {k: v for k, v in r["phases"].items() if not k.endswith("detail")}}
                if cfg == "C2" and not a.no_e2e:
                    item["e2e"] = ex.host_image(a.extra_steps, a.warmup)
                ex.close()
                extras[cfg] = item
            except Exception as e:  # an extra never sinks the main line
                extras[cfg] = {"error": repr(e)[:300]}
                torch.cuda.empty_cache()

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_baseline(w)
        cpu["cores_available"] = os.cpu_count()

    if rank == 0:
        out = {
            "metric": METRIC, "value": main_res["value"], "unit": "GB/s", "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": main_res["ms_per_step"], "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": w.name, "payload_bytes_per_gpu": S, "n_buffers": len(w.buffers),
                       "n_chunks": n_chunks, "fill": a.kind,
                       "image": "device-resident (HBM), reused across steps",
                       "step": ("checkpoint -> release every handle (restart) -> restore re-creates them" if snap.restart
                                else "checkpoint -> restore (rebind)") + (" ; status all-reduce of the global snapshot "
                                                                         "(coordinated, real outcome)" if world > 1 else ""),
                       "l2": ("inputs larger than L2" if S > L2_BYTES
                              else "inputs smaller than L2: L2 flushed (252 MB write) before every timed step"),
                       "parallelism": f"independent snapshot per rank, {world} rank(s)"},
            "roofline": main_res["roofline"],
            "phases": main_res["phases"],
            "verified": main_res["verified"],
            "gpu_launches": main_res["gpu_launches"],
            "clocks": main_res["clocks"],
            "cpu_baseline": cpu,
            "e2e": e2e,
            "extras": extras,
        }
        print(json.dumps(out))
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
