"""bench.py end to end on a B200 with the small config (the driver runs the C2 line): the JSON
line carries the contract's keys (roofline with the measured peak, cpu_baseline with the host
description, e2e with its copied bytes, gpu_launches, clocks), the oracle reorder timing, K=32,
and the single-GPU shard simulation."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_line_tiny():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--config", "tiny", "--K", "32",
                        "--extra-K", "128", "--steps", "3", "--warmup", "3", "--cpu-seconds", "1",
                        "--e2e-steps", "1", "--simulate-world", "2", "--panel-rows", "16", "--dense-min", "2"],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads(r.stdout.strip().splitlines()[-1])
    assert d["metric"] == "SpMM+SDDMM GFLOP/s (2*nnz*K per op)" and d["value"] > 0 and d["n_gpus"] == 1
    assert d["gpu_launches"] >= 3 * 2 and d["steps"] == 3 and d["warmup"] == 3
    roof = d["roofline"]
    assert roof["bound"] == "hbm" and 0 < roof["frac"] and roof["peak"] > 0 and "traffic" in roof
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["host"]["logical_cpus"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert "sm_mhz" in d["clocks"]
    assert d["preprocess"]["oracle"]["seconds"] > 0
    assert d["extra_K"]["128"]["value"] > 0
    sim = d["shard_simulation"]
    assert sim["world"] == 2 and len(sim["per_shard_ms"]) == 2 and sum(sim["per_shard_nnz"]) == d["config"]["nnz"]
