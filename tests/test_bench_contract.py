"""bench.py's JSON line (the driver contract): one line on stdout with the metric, the
whole-job value, the timing protocol fields, the roofline and cpu_baseline objects, the
end-to-end number and the clocks.  The reference arm (the CPU oracle) runs on CPU; the
mdh arm needs the GPU."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
             "vs_baseline", "dtype", "data", "config", "e2e"}


def _run(args, timeout):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:]
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _run(["--impl", "reference", "--workload", "dot_f32", "--steps", "1", "--warmup", "1"], 600)
    assert BASE_KEYS <= set(d), set(d) ^ BASE_KEYS
    assert d["impl"] == "reference" and d["config"]["workload"] == "dot_f32"
    assert d["warmup"] >= 3                         # W ≥ 3 is enforced
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0


@pytest.mark.gpu
def test_mdh_arm_line():
    d = _run(["--no-suite", "--no-cpu-baseline", "--steps", "3", "--warmup", "3"], 900)
    assert BASE_KEYS <= set(d), set(d) ^ BASE_KEYS
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3 and d["value"] > 0
    assert d["config"]["workload"] == "matmul_bf16" and "l2" in d["config"]
    rl = d["roofline"]
    assert rl["bound"] == "tensor" and rl["unit"] == "TFLOP/s" and 0 < rl["frac"] <= 1.2
    assert abs(rl["frac"] - rl["achieved"] / rl["peak"]) < 1e-9
    e = d["e2e"]
    assert e["h2d_bytes_per_step"] == 2 * 4096 * 4096 * 2 and e["d2h_bytes_per_step"] == 4096 * 4096 * 4
    assert 0 < e["value"] < d["value"]
    assert d["gpu_launches"] >= d["steps"]
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= set(d["clocks"])
    assert d["parity_sample"]["max_rel_err"] <= 1e-2
