"""bench.py (our arm) keeps the driver's JSON contract on a B200: one line with the metric, the
roofline object (HBM-bound consume kernel, achieved / peak / frac / traffic), clocks, gpu_launches,
e2e with the bytes copied, and the timing rules (warmup >= 3 by default, K steps)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_line_contract():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "3",
                        "--no-slowdown", "--no-injection", "--no-cpu-baseline"],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [json.loads(l) for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = lines[0]
    assert d["metric"].startswith("warp-instr records/sec") and d["unit"] == "records/s"
    assert d["value"] > 1e9 and d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] >= 3
    assert d["scaling"] == "weak" and d["data"] == "synthetic" and d["config"]["workload"].startswith("c3")
    rf = d["roofline"]
    assert rf["bound"] == "hbm" and rf["unit"] == "GB/s" and 0 < rf["frac"] < 1.2
    assert abs(rf["frac"] - rf["achieved"] / rf["peak"]) < 1e-9
    assert rf["traffic"] is None or rf["traffic"] >= rf["algorithmic_bytes_per_launch"]
    assert d["gpu_launches"] > 0 and "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
