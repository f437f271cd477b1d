"""-m "not gpu": the driver's bench.py contract for the reference arm, which for this
tier is the oracle on the host cores. Runs C1 (configs[0]) with one
process and under torchrun with two ranks (rank 0 alone runs and prints; the other
rank exits 0 without work)."""
import json
import os
import socket
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
        "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _json_lines(out):
    return [json.loads(l) for l in out.splitlines() if l.startswith("{")]


def _check_line(d, n_gpus):
    assert KEYS <= set(d), KEYS - set(d)
    assert d["impl"] == "reference" and d["n_gpus"] == n_gpus
    assert d["steps"] == 1 and d["warmup"] == 3
    assert d["unit"] == "GB/s" and d["higher_is_better"] is True and d["value"] > 0
    assert d["config"]["workload"].startswith("C1") and d["config"]["payload_bytes_per_gpu"] == 3 * 1048576
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        assert d["metric"] == json.load(f)["metric"]


def test_reference_arm_one_process():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--config", "C1", "--steps", "1",
                        "--warmup", "3"], cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1
    _check_line(lines[0], 1)


def test_reference_arm_two_ranks_rank0_prints_once():
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py",
                        "--gpus", "2", "--impl", "reference", "--config", "C1", "--steps", "1", "--warmup", "3"],
                       cwd=ROOT, capture_output=True, text=True, timeout=300, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1
    _check_line(lines[0], 2)


def test_host_ram_check_and_meminfo(monkeypatch):
    """The e2e leg pins one image per local rank: bench.host_ram_check compares that
    with MemAvailable (70 % of it), which bench.meminfo_available reads from
    /proc/meminfo (C4 at 8 ranks needs ~512 GiB: scaled down)."""
    sys.path.insert(0, ROOT)
    import bench
    avail = bench.meminfo_available()
    assert avail > 0
    monkeypatch.setattr(bench, "meminfo_available", lambda: 196 << 30)
    fits, need, av = bench.host_ram_check(68_719_476_448, 8)
    assert not fits and need == 8 * 68_719_476_448 and av == 196 << 30
    fits, need, _ = bench.host_ram_check(5_350_180_722, 8)
    assert fits and need == 8 * 5_350_180_722
    monkeypatch.setattr(bench, "meminfo_available", lambda: 0)  # unknown: assume it fits
    assert bench.host_ram_check(1 << 40, 8)[0]
