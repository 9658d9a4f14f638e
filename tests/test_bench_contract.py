"""bench.py contract on the CPU: the reference arm's JSON line (keys, types,
units, its e2e block) on a tiny config, and the helpers the GPU arm's
roofline blocks are computed with (SURVEY 8(d) bytes_alg, gather bytes)."""
import json
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import gen  # noqa: E402


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config",
                        "c1_uniform1024", "--steps", "3", "--warmup", "3"], capture_output=True, text=True,
                       timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "impl", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["metric"] == bench.METRIC
    assert d["unit"] == "GFLOP/s" and d["higher_is_better"] is True
    assert d["steps"] == 3 and d["warmup"] == 3 and d["n_gpus"] == 1
    assert d["config"]["workload"] == "c1_uniform1024" and d["config"]["J"] == 32
    A_h, J = gen.config("c1_uniform1024")
    # value = 2 nnz J / t over the sampled rows (here: all of them)
    assert d["config"]["sample_nnz"] == A_h.nnz
    assert abs(d["value"] - 2 * A_h.nnz * J / (d["ms_per_step"] * 1e-3) / 1e9) <= 1e-6 * d["value"]
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"] == {"value": d["value"], "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


def test_algorithmic_bytes_and_gather_roofline():
    # bytes_alg = nnz * (4 + 4) + U * J * 4 + I * J * 4 on a hand-made CSR
    rp = np.array([0, 2, 2, 5], np.int64)
    ci = np.array([0, 3, 0, 1, 3], np.int32)
    A = gen.CSR(3, 5, rp, ci, np.ones(5, np.float32))
    b, U = bench.algorithmic_bytes(A, 8)
    assert U == 3 and b == 5 * 8 + 3 * 8 * 4 + 3 * 8 * 4
    g = bench.gather_roofline("c2_rmat20", 1000, 128, 1, 0.5)
    assert g["bytes_per_launch"] == 1000 * 128 * 4
    assert abs(g["achieved"] - 1000 * 128 * 4 / 0.5e-3 / 1e9) < 1e-9
    assert g["ceiling"] == bench.GATHER_CEILING["c2_rmat20"][0] and abs(g["frac"] - g["achieved"] / g["ceiling"]) < 1e-12
    assert "ceiling" not in bench.gather_roofline("no_such_config", 10, 32, 1, 1.0)
    # the FP32 CUDA-core peak is SMs x 128 FMA/clk x 2 x clock
    assert bench.fp32_peak_tflops() > 10.0


def test_traffic_is_only_used_for_its_own_sources():
    """roofline.traffic comes from profiles/traffic.json only when its source
    hash equals the sources bench.py runs; otherwise None with the reason."""
    t = bench.ncu_traffic("c2_rmat20", 128)
    with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
        rec = json.load(f)
    if rec["src_hash"] == bench.src_hash():
        assert isinstance(t[0], int) and t[0] > 0
    else:
        assert t[0] is None and "stale" in t[1]
    assert bench.ncu_traffic("no_such_config", 1)[0] is None
