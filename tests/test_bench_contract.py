"""bench.py keeps the driver's JSON-line contract: the reference arm (the fp64
oracle on the host cores) on CPU, and our arm at quick sizes on a B200."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]


def run_bench(*args, timeout=600, torchrun_env=True):
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    if not torchrun_env:
        for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK"):
            env.pop(k, None)
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
    assert d["in_hbm"]["value"] > 0 and "slowdown_pct_vs_in_hbm" in d
    M, N, K = d["config"]["M"], d["config"]["N"], d["config"]["K"]
    assert d["e2e"]["h2d_bytes_per_step"] >= 4 * (M * K + K * N)        # every A/B byte crosses PCIe
    assert d["e2e"]["d2h_bytes_per_step"] == 4 * M * N
    assert d["gpu_launches"] > 0
    rl = d["roofline"]
    assert rl["bound"] == "tensor" and 0 < rl["frac"] < 1.2 and rl["peak"] > 0
    assert rl["kernel"] == "nu::leaf::x3::leaf_x3_kernel" and rl["launches_timed"] > 0
    er = d["e2e_roofline"]
    assert er["bound"] in ("tensor", "pcie_h2d", "pcie_d2h") and 0 < er["frac"] < 1.2
    assert d["staging"]["pcie_measured"]["h2d_gbs"] > 1
    assert d["parity"]["bitwise_in_hbm_vs_out_of_core"] and d["parity"]["bitwise_tree_vs_leaf"]
    assert d["parity"]["oracle_ok"] and d["cpu_baseline"]["kind"] == "oracle"
    assert d["cpu_baseline"]["single_core_value"] > 0 and d["cpu_baseline"]["numa_nodes"] >= 1
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]
    assert d["cfg2_in_hbm_tflops"] > 0 and "slowdown_pct_vs_cfg2_in_hbm" in d
    assert 0 <= d["runtime_overhead"]["plan_pct_of_step"] < 100
    assert 0 < d["breakdown"]["compute_pct"] <= 100
    assert set(d["in_hbm"]["split_variants_tflops"]) == {"npass4", "npass1"}


@pytest.mark.gpu
def test_hotspot_quick_json_line():
    """--config hotspot: the NEXT-3 line with its alu roofline, the out-of-core
    roofline from the link rates measured in the same run, and a stream breakdown."""
    d = run_bench("--config", "hotspot", "--quick", "--steps", "2", "--warmup", "3")
    assert d["unit"] == "Gcell-updates/s" and d["value"] > 0 and d["in_hbm"]["value"] > 0
    assert d["roofline"]["bound"] == "alu" and 0 < d["roofline"]["frac"] < 1
    er = d["e2e_roofline"]
    assert er["bound"] in ("pcie_h2d", "pcie_d2h", "in_hbm") and 0 < er["frac"] < 1.2
    assert set(er["terms"]) == {"pcie_h2d", "pcie_d2h", "in_hbm"}
    assert d["e2e"]["pcie_measured"]["bidir_h2d_gbs"] > 1
    assert d["breakdown"]["compute_busy_ms"] > 0 and d["breakdown"]["h2d_busy_ms"] > 0
    assert d["parity"]["bitwise_in_hbm_vs_out_of_core"] and d["parity"]["oracle_ok"]


@pytest.mark.gpu
def test_ours_spawns_ranks_for_gpus_n():
    """`python bench.py --gpus 4` outside torchrun starts the 4 ranks itself
    (here 4 processes share the one GPU: --device-mod 1, gloo)."""
    d = run_bench("--gpus", "4", "--quick", "--steps", "2", "--warmup", "3", "--device-mod", "1",
                  "--dist-backend", "gloo", "--no-cpu-baseline", timeout=900, torchrun_env=False)
    assert d["n_gpus"] == 4 and d["value"] > 0 and d["config"]["workload"].startswith("cfg4")


def test_gpus_mismatch_with_world_size_fails_loudly():
    """--gpus N under a launcher that started a different number of ranks."""
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2"], capture_output=True,
                       text=True, timeout=120, cwd=ROOT, env=env)
    assert r.returncode == 2 and "WORLD_SIZE=1" in r.stderr


def test_ooc_roofline_terms():
    """S§8(d): R = min(P_eff, BW_h2d * I_h2d, BW_d2h * I_d2h), I_e = flops / bytes on edge e."""
    sys.path.insert(0, ROOT)
    import bench
    pcie = {"bidir_h2d_gbs": 50.0, "bidir_d2h_gbs": 51.0}
    flops = 2.0 * 32768 ** 3
    r = bench.ooc_roofline(flops, 8 << 30, 4 << 30, 344.0, pcie)
    assert r["intensity_flop_per_byte"] == {"h2d": 8192.0, "d2h": 16384.0}
    assert abs(r["terms"]["pcie_h2d"] - 50e9 * 8192 / 1e12) < 1e-3
    assert r["bound"] == "tensor" and r["peak"] == 344.0
    r5 = bench.ooc_roofline(2.0 * 1048576 * 4096 * 4096, 16 << 30, 16 << 30, 344.0, pcie)
    assert r5["bound"] == "pcie_h2d" and abs(r5["peak"] - 50e9 * 2048 / 1e12) < 1e-2
    assert bench.ooc_roofline(1e12, 0, 0, 344.0, pcie)["bound"] == "tensor"   # in-HBM: no edges
