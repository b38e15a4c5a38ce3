"""bench.py's JSON-line contract (the driver parses it): the keys, their types
and the invariants between them, for the oracle arm on CPU and for the CUDA arm
on a GPU (c1: seconds to run)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
             "vs_baseline", "dtype", "data", "config", "e2e"}


def run_bench(*args):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def check_common(d, steps, warmup):
    assert BASE_KEYS <= set(d), BASE_KEYS - set(d)
    assert d["metric"] == "Munknowns/s fp64/fp32 and % of HBM roofline at 1/2/4/8 B200"
    assert d["unit"] == "Munknowns/s" and d["higher_is_better"] is True
    assert d["steps"] == steps and d["warmup"] == warmup and d["n_gpus"] == 1
    assert d["value"] > 0 and d["ms_per_step"] > 0
    assert d["scaling"] in ("weak", "strong")
    assert d["data"].startswith("synthetic")
    assert d["config"]["workload"] == "c1" and d["config"]["n"] == 1024 and d["config"]["m"] == 1
    e = d["e2e"]
    assert {"value", "unit", "h2d_bytes_per_step", "d2h_bytes_per_step"} <= set(e)


def test_reference_arm_contract():
    """--impl reference: the CPU oracle on this host, its cpu_baseline block and a
    zero-copy e2e (runs without a GPU)."""
    d = run_bench("--impl", "reference", "--config", "c1", "--steps", "2", "--warmup", "1")
    check_common(d, 2, 1)
    assert d["impl"] == "reference"
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"]["value"] == d["value"] and d["e2e"]["h2d_bytes_per_step"] == 0


@pytest.mark.gpu
def test_cuda_arm_contract():
    """The CUDA arm: roofline (algorithmic bytes over the measured peak), the
    oracle timed beside it, the host-buffer e2e with its copy volumes, the clocks
    sampled under load, and the kernel launch count."""
    d = run_bench("--config", "c1", "--steps", "5", "--warmup", "3")
    check_common(d, 5, 3)
    assert d.get("impl", "ours") == "ours" and d["dtype"] == "f64"
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and r["peak"] > 1000
    assert 0 < r["frac"] <= 1.2 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-9
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] > 0
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] == 4 * 1024 * 8 and e["d2h_bytes_per_step"] == 1024 * 8
    c = d["clocks"]
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= set(c)
    assert d["gpu_launches"] >= 5
    assert d["parity"]["max_rel_err"] <= 1e-10
