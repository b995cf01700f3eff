"""bench.py keeps the driver contract: one JSON line with the required keys, for the product
arm (GPU, small grid) and for the reference arm (the CPU oracle)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "e2e"}


def _run(*args, timeout=900):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip().startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_contract():
    d = _run("--impl", "reference", "--n", "48", "--nt", "20", "--steps", "1", "--warmup", "3")
    assert BASE <= set(d) and d["impl"] == "reference" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["config"]["workload"].startswith("C2 acoustic")


@pytest.mark.gpu
def test_product_arm_contract():
    d = _run("--n", "96", "--nt", "40", "--steps", "3", "--warmup", "3", "--no-extras")
    assert BASE <= set(d) and d["value"] > 0 and d["n_gpus"] == 1
    assert {"gpu_launches", "roofline", "clocks", "cpu_baseline"} <= set(d) and d["gpu_launches"] > 0
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and 0 < r["frac"] == pytest.approx(r["achieved"] / r["peak"], rel=1e-3)
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle"
    assert d["config"]["workload"].startswith("C2 acoustic 96x96x96")
