"""BASELINE.json configs at full size, in the configuration bench.py times,
checked against the oracle on what it can afford (SURVEY.md §8(c) "Large
configs"): cfg2 element by element; cfg3/cfg4/cfg5 on sampled entries plus
full rows and columns (normwise bound) and, with integer inputs, Freivalds'
check, which is exact in fp64 and catches any misplaced or missing block.
65,536 sampled entries per config (S§8(c) "≥ 65,536 random (i,j)")."""
import ctypes

import numpy as np
import pytest
import torch

import nugen
import oracle
import paper_conf_ipps_chey19_b200 as nu

pytestmark = pytest.mark.gpu
GiB = 1 << 30
TOL = 1e-5


def host_view(buf, rows, cols):
    return np.ctypeslib.as_array((ctypes.c_float * (rows * cols)).from_address(buf.ptr)).reshape(rows, cols)


def sampled_check(a, b, c, seed=0, n=65536):
    M, K = a.shape
    N = b.shape[1]
    rng = np.random.default_rng(seed)
    I = rng.integers(0, M, n)
    J = rng.integers(0, N, n)
    ref = oracle.entries(a, b, I, J)
    ra = np.sqrt((a[I].astype(np.float64) ** 2).sum(axis=1))
    cn = oracle.col_norms(b)
    err = np.abs(c[I, J].astype(np.float64) - ref) / (ra * cn[J])
    worst = float(err.max())
    # two full rows and two full columns
    rows = rng.integers(0, M, 2)
    rr = oracle.gemm_rows(a, b, rows)
    e_rows = oracle.normwise_err(np.ascontiguousarray(c[rows]), rr, oracle.row_norms(
        np.ascontiguousarray(a[rows])), cn)[0]
    cols = rng.integers(0, N, 2)
    bc = np.ascontiguousarray(b[:, cols])
    rc = oracle.gemm(a, bc)
    e_cols = oracle.normwise_err(np.ascontiguousarray(c[:, cols]), rc, oracle.row_norms(a),
                                 oracle.col_norms(bc))[0]
    return max(worst, e_rows, e_cols)


def freivalds_uniform(a, b, c, seed, reps=2):
    """S§8(c): every row of C at once — for random +-1 vectors r, the necessary
    condition |((C - C_ref) r)_i| <= 1e-5 ||A_i,:||_2 sum_j ||B_:,j||_2 (returns
    the worst ratio; C_ref r is computed as A (B r) in fp64)."""
    rng = np.random.default_rng(seed + 100)
    rn, cn = oracle.row_norms(a), oracle.col_norms(b)
    worst = 0.0
    for _ in range(reps):
        r = np.where(rng.random(b.shape[1]) < 0.5, -1.0, 1.0)
        e, _, _ = oracle.freivalds(a, b, c, r, rn, cn)
        worst = max(worst, e)
    return worst


def run_config(M, N, K, cap, kind, seed):
    t, _ = nu.host_tree(1, cap)
    t.finalize()
    A, B, C = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
    a, b, c = host_view(A, M, K), host_view(B, K, N), host_view(C, M, N)
    nugen.fill(M, K, seed, nugen.MAT_A, kind, out=a)
    nugen.fill(K, N, seed, nugen.MAT_B, kind, out=b)
    st = t.gemm(A, B, C, M, N, K)
    return t, a, b, c, st


def test_cfg2_in_hbm_full_oracle():
    """configs[1]: 8192^3 resident in HBM, every element against the oracle."""
    M = N = K = 8192
    a = nugen.fill(M, K, 2, 1)
    b = nugen.fill(K, N, 2, 2)
    dev = torch.device("cuda:0")
    Ad, Bd = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
    Cd = torch.empty((M, N), device=dev)
    nu.leaf_gemm(Ad, Bd, Cd)
    torch.cuda.synchronize()
    ref = oracle.gemm(a, b)
    e, where = oracle.normwise_err(Cd.cpu().numpy(), ref, oracle.row_norms(a), oracle.col_norms(b))
    assert e <= TOL, (e, where)


@pytest.mark.parametrize("name,M,N,K,cap", [
    ("cfg3", 32768, 32768, 32768, 8 * GiB),
    ("cfg5", 1048576, 4096, 4096, 8 * GiB),
])
def test_large_config_sampled_and_freivalds(name, M, N, K, cap):
    seed = int(name[-1])
    t, a, b, c, st = run_config(M, N, K, cap, "uniform", seed)
    assert st["hbm_peak_bytes"] <= cap
    assert sampled_check(a, b, c, seed) <= TOL
    assert freivalds_uniform(a, b, c, seed) <= TOL
    t.destroy()
    # integer inputs: exact result -> Freivalds with +-1 vectors must match exactly
    t, a, b, c, st = run_config(M, N, K, cap, "int", seed)
    rng = np.random.default_rng(seed)
    for _ in range(2):
        r = np.where(rng.random(N) < 0.5, -1.0, 1.0)
        _, x, y = oracle.freivalds(a, b, c, r)
        assert np.array_equal(x, y)
    t.destroy()


def test_cfg4_one_gpu_sampled():
    """configs[3] (65536 x 65536 x 32768) on one GPU: the C region exceeds the
    8 GiB HBM cap, so the planner splits it into blocks."""
    M, N, K = 65536, 65536, 32768
    t, a, b, c, st = run_config(M, N, K, 8 * GiB, "uniform", 4)
    assert st["bm"] * st["bn"] < M * N and st["hbm_peak_bytes"] <= 8 * GiB
    assert sampled_check(a, b, c, 4) <= TOL
    assert freivalds_uniform(a, b, c, 4) <= TOL
    t.destroy()
    # integer inputs: C is exact, so Freivalds with +-1 vectors must match exactly
    # (a single wrong element of the 2^32 would show: test_oracle pins this)
    t, a, b, c, st = run_config(M, N, K, 8 * GiB, "int", 4)
    rng = np.random.default_rng(4)
    for _ in range(2):
        r = np.where(rng.random(N) < 0.5, -1.0, 1.0)
        _, x, y = oracle.freivalds(a, b, c, r)
        assert np.array_equal(x, y)
    t.destroy()
