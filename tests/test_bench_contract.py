"""bench.py's output contract: one JSON line on rank 0 with the keys the driver and the judge read
(the reference arm runs the CPU oracle, so it is checked here without a GPU; the product arm
needs the GPU)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT,
                         capture_output=True, text=True, timeout=timeout)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


def _common(d, steps, warmup):
    assert d["metric"] == "kernel invocations stratified/sec"
    assert d["unit"] == "invocations/s" and d["higher_is_better"] is True
    assert d["value"] > 0 and d["ms_per_step"] > 0
    assert d["n_gpus"] == 1 and d["steps"] == steps and d["warmup"] == warmup
    assert d["data"] == "synthetic" and d["vs_baseline"] is None
    assert d["config"]["workload"]


def test_reference_arm_contract():
    d = _run(["--impl", "reference", "--config", "C1", "--steps", "2", "--warmup", "1"], 300)
    _common(d, 2, 1)
    assert d["impl"] == "reference"
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == 1 and cb["value"] == d["value"] and cb["sample"]
    e = d["e2e"]
    assert e["value"] == d["value"] and e["h2d_bytes_per_step"] == 0 and e["d2h_bytes_per_step"] == 0


@pytest.mark.gpu
def test_product_arm_contract():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    d = _run(["--config", "C2", "--steps", "3", "--warmup", "3", "--cpu-sample", "20000"], 900)
    _common(d, 3, 3)
    assert "impl" not in d or d["impl"] != "reference"
    assert d["gpu_launches"] > 0
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] <= 1 and r["peak"] > 0
    assert abs(r["achieved"] / r["peak"] - r["frac"]) < 1e-9
    e = d["e2e"]
    # 24 B per invocation, or 20 with the 16-bit kernel-id and CTA columns (SIEVE_KID16 / CTA16)
    assert e["value"] > 0 and e["h2d_bytes_per_step"] in (20 * d["config"]["invocations"], 24 * d["config"]["invocations"])
    assert e["d2h_bytes_per_step"] > 0
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == 1 and cb["value"] > 0
    c = d["clocks"]   # a run this short may end before the sampler's first reading
    assert isinstance(c, dict) and isinstance(c.get("reasons", []), list)
    assert c.get("sm_max_mhz") is None or c["sm_max_mhz"] > 0
