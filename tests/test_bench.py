"""bench.py contract: the JSON line the driver parses (both arms).

CPU: the reference arm (the oracle on host cores, bounded sample) prints one
line with the contract's keys.  GPU: our arm on class S (fast) prints the
contract's keys, a positive value, the roofline/cpu_baseline/e2e/clocks
objects, and a result equal to NPB's class-S verification sums."""
import json
import os
import subprocess
import sys

import pytest

from ep_workloads import NPB_EPS

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
        "scaling", "vs_baseline", "dtype", "data", "config", "e2e"}
SX_S, SY_S = -3.247834652034740e3, -6.958407078382297e3   # NPB ep.f verify, class S


def run_bench(*args, timeout=600):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_reference_arm_contract():
    d = run_bench("--impl", "reference", "--cls", "S", "--steps", "2", "--warmup", "3", "--ref-batches", "16")
    assert d["impl"] == "reference"
    assert KEYS <= set(d)
    assert d["value"] > 0 and d["unit"] == "Mops/s" and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["config"]["workload"].startswith("NPB EP class S")


@pytest.mark.gpu
def test_our_arm_contract_class_S():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    d = run_bench("--cls", "S", "--steps", "5", "--warmup", "3", "--cpu-budget", "1")
    assert KEYS <= set(d) and d["n_gpus"] == 1 and d["dtype"] == "f64"
    assert d["value"] > 0 and d["gpu_launches"] >= 5
    rf = d["roofline"]
    assert rf["bound"] == "alu" and 0 < rf["frac"] <= 1 and rf["peak"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["value"] > 0 and d["e2e"]["d2h_bytes_per_step"] == 104
    assert "sm_mhz" in d["clocks"]
    res = d["result"]
    assert abs((res["sx"] - SX_S) / SX_S) <= NPB_EPS and abs((res["sy"] - SY_S) / SY_S) <= NPB_EPS
