"""The driver contract of bench.py (one GPU): one JSON line with the keys the
round-end driver and the judge read, values consistent with each other and
with the oracle's statistics of the named workload.  Uses the tiny space so
it runs in seconds; the headline runs are the driver's own."""
from __future__ import annotations

import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

pytestmark = pytest.mark.gpu


def _run(*args):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT,
                         capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_json_line_contract():
    import beast_inputs
    import oracle
    d = _run("--workload", "widened256_k40c", "--steps", "5", "--warmup", "3", "--no-sweep", "--no-ir")
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "e2e", "gpu_launches",
              "clocks", "cpu_baseline", "write_out"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["steps"] == 5 and d["warmup"] == 3
    assert d["higher_is_better"] is True and d["unit"] == "points/s"
    ref = oracle.nest(beast_inputs.named("widened256_k40c"))
    assert d["config"]["n_canon"] == sum(ref["visits"])
    assert d["config"]["survivors"] == ref["survivors"]
    assert abs(d["value"] - d["config"]["n_canon"] / (d["ms_per_step"] / 1e3)) <= 1e-6 * d["value"]
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 2 and abs(r["achieved"] / r["peak"] - r["frac"]) < 1e-9
    e = d["e2e"]
    assert e["d2h_bytes_per_step"] >= 16 * d["config"]["survivors"] and e["value"] > 0
    assert d["write_out"]["bytes_per_launch"] == 16 * d["config"]["survivors"]
    assert d["gpu_launches"] > 0
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] >= 1 and c["value"] > 0 and c["single_thread"]["value"] > 0
    # count timed on its own, N_space as context, the oracle
    # over configs[0..2] with the CPU model, the measured-scan fraction
    assert d["count"]["value"] > 0 and d["count"]["ms_per_step"] > 0
    assert [x["config"][:10] for x in c["configs"]] == ["configs[0]", "configs[1]", "configs[2]"]
    assert c["configs"][1]["points"] == 2_096_997_743 and c["configs"][2]["spaces"] == 12
    assert int(c["n_space"]) > d["config"]["n_canon"] and c["cpu"]["model_name"]
    assert 0 < r["frac_measured_scan"] < r["frac"]
    assert d["sharded_resident"] is None and d["replicas"]["ranks_agree"] is True
    assert e["h2d_bytes_per_step"] == 0


def test_bench_reference_arm():
    d = _run("--impl", "reference", "--workload", "widened256_k40c", "--steps", "3", "--warmup", "3")
    assert d["impl"] == "reference" and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"
    g = _run("--workload", "widened256_k40c", "--steps", "3", "--warmup", "3", "--no-sweep", "--no-ir",
             "--no-cpu-baseline")
    assert d["config"] == g["config"]                  # the driver's same-config check


def test_bench_gpus_more_than_visible_fails_loudly():
    """--gpus N without a launcher starts N ranks itself; with fewer GPUs than
    N visible it must fail, not measure one GPU and print n_gpus 1."""
    import torch
    n = torch.cuda.device_count()
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(n + 1), "--steps", "3"],
                         cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert out.returncode != 0 and "visible" in out.stderr
    assert not [l for l in out.stdout.splitlines() if l.startswith("{")]
