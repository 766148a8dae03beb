"""bench.py keeps the driver's JSON-line contract: the reference arm (the fp64
oracle on the host cores) on CPU, and our arm at quick sizes on a B200."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]


def run_bench(*args, timeout=600):
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True,
                       text=True, timeout=timeout, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.strip().splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_json_line():
    d = run_bench("--impl", "reference", "--quick", "--steps", "2", "--warmup", "0", "--ref-step-s", "0.2",
                  timeout=300)
    assert d["impl"] == "reference" and d["metric"] == METRIC and d["unit"] == "TFLOP/s"
    assert d["value"] > 0 and d["higher_is_better"] is True and d["steps"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"] == {"value": d["value"], "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    assert d["config"]["workload"].startswith("cfg3")


@pytest.mark.gpu
def test_ours_quick_json_line():
    d = run_bench("--quick", "--steps", "2", "--warmup", "3", "--cpu-budget", "1")
    assert d["metric"] == METRIC and d["unit"] == "TFLOP/s" and d["n_gpus"] == 1
    assert d["value"] > 0 and d["e2e"]["value"] > 0 and d["e2e"]["unit"] == "TFLOP/s"
    M, N, K = d["config"]["M"], d["config"]["N"], d["config"]["K"]
    assert d["e2e"]["h2d_bytes_per_step"] >= 4 * (M * K + K * N)        # every A/B byte crosses PCIe
    assert d["e2e"]["d2h_bytes_per_step"] == 4 * M * N
    assert d["gpu_launches"] > 0
    rl = d["roofline"]
    assert rl["bound"] == "tensor" and 0 < rl["frac"] < 1.1 and rl["peak"] > 0
    er = d["e2e_roofline"]
    assert er["bound"] in ("tensor", "pcie_h2d", "pcie_d2h") and 0 < er["frac"] < 1.1
    assert d["staging"]["pcie_measured"]["h2d_gbs"] > 1
    assert d["parity"]["bitwise_in_hbm_vs_out_of_core"] and d["parity"]["bitwise_tree_vs_leaf"]
    assert d["parity"]["oracle_ok"] and d["cpu_baseline"]["kind"] == "oracle"
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]
    assert d["cfg2_in_hbm_tflops"] > 0 and "slowdown_pct_vs_cfg2_in_hbm" in d
