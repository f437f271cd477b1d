"""Box probe: host facts + pinned PCIe copy bandwidth + HBM copy (torch plumbing only).

Writes gpurun_out/probe_box.json. Used to fix the PCIe roofline denominators.
"""
import json, os, subprocess, time
import torch

out = {}
def sh(c):
    try:
        return subprocess.run(c, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e:
        return str(e)
out["nproc"] = os.cpu_count()
out["lscpu"] = sh("lscpu | head -30")
out["free_g"] = sh("free -g")
out["nvidia_smi"] = sh("nvidia-smi --query-gpu=name,pci.bus_id,memory.total,clocks.max.sm,pcie.link.gen.max,pcie.link.width.max,pcie.link.gen.current --format=csv")
out["topo"] = sh("nvidia-smi topo -m")
out["numa"] = sh("numactl -H 2>/dev/null | head -5; cat /sys/bus/pci/devices/*/numa_node 2>/dev/null | sort | uniq -c")
dev = torch.device("cuda:0")
torch.cuda.init()
res = {}
for mb in (32, 64, 256, 1024):
    n = mb << 20
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    h.fill_(1)
    d = torch.empty(n, dtype=torch.uint8, device=dev)
    s = torch.cuda.Stream()
    for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))):
        with torch.cuda.stream(s):
            for _ in range(3): fn()
            s.synchronize()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            reps = 10
            e0.record(s)
            for _ in range(reps): fn()
            e1.record(s); e1.synchronize()
            res[f"{name}_{mb}MiB_GBs"] = n * reps / (e0.elapsed_time(e1) * 1e-3) / 1e9
    # bidirectional
    s2 = torch.cuda.Stream()
    h2 = torch.empty(n, dtype=torch.uint8, pin_memory=True); d2 = torch.empty(n, dtype=torch.uint8, device=dev)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(5):
        with torch.cuda.stream(s): d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    torch.cuda.synchronize()
    res[f"bidir_{mb}MiB_GBs_each"] = n * 5 / (time.perf_counter() - t0) / 1e9
    del h, d, h2, d2
a = torch.empty(1 << 30, dtype=torch.uint8, device=dev); b = torch.empty_like(a)
for _ in range(3): b.copy_(a)
torch.cuda.synchronize()
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10): b.copy_(a)
e1.record(); e1.synchronize()
res["hbm_copy_GBs_rw"] = 2 * (1 << 30) * 10 / (e0.elapsed_time(e1) * 1e-3) / 1e9
# pin cost
t0 = time.perf_counter(); hp = torch.empty(4 << 30, dtype=torch.uint8, pin_memory=True); res["pin_4GiB_s"] = time.perf_counter() - t0
out["bw"] = res
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe_box.json", "w"), indent=1)
print(json.dumps(res, indent=1))
