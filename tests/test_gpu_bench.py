"""bench.py's driver contract (the task's measurement rules):
one JSON line on rank 0 with the metric BASELINE.json names, the workload, device-timed
value, roofline / e2e / clocks / gpu_launches objects; --gpus N without torchrun re-runs
itself as N ranks (here over the host communicator, the N ranks sharing one GPU).
Runs the Enron-shaped config (configs[2], 54M nonzeros) to keep the test short."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run_bench(*args, timeout=900):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:]
    return json.loads(lines[0])


def test_bench_contract_one_gpu():
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        metric = json.load(f)["metric"]
    d = run_bench("--config", "enron", "--steps", "3", "--warmup", "3", "--no-cpu-baseline",
                  "--no-streaming-probe")
    assert d["metric"] == metric and d["unit"] == "s" and d["higher_is_better"] is False
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3
    assert d["value"] > 0 and abs(d["ms_per_step"] - 1e3 * d["value"]) <= 1e-6 * d["ms_per_step"]
    assert d["dtype"] == "f64" and d["config"]["workload"] == "enron"
    assert d["gpu_launches"] > 0
    r = d["roofline"]
    for k in ("bound", "achieved", "peak", "unit", "frac", "traffic"):
        assert k in r, k
    assert r["bound"] == "hbm" and 0 < r["frac"] < 1 and r["unit"] == "GB/s"
    assert r["frac"] == pytest.approx(r["achieved"] / r["peak"], rel=1e-9)
    e = d["e2e"]
    assert e["value"] > d["value"] and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]


def test_bench_two_ranks_relaunch():
    d = run_bench("--config", "enron", "--steps", "2", "--warmup", "3", "--gpus", "2", "--comm", "host",
                  "--no-cpu-baseline", "--no-e2e", "--no-streaming-probe")
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["workload"] == "enron"
