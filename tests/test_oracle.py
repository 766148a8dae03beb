"""Pins for the oracle (SURVEY.md §8(c) "What pins each part").

The paper prints no worked numeric example for dense MM, so O1 is pinned to
brute force on tiny hand cases, closed forms, and a library routine
(numpy.matmul / BLAS dgemm, an independent implementation).  O2 (Listing 3
recursion) is pinned to O1 bitwise on integer inputs.  The checkers are pinned
by planting known errors.
"""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import nugen
import oracle
from conftest import load_golden


def f32(x):
    return np.ascontiguousarray(x, dtype=np.float32)


@pytest.mark.parametrize("name", ["mm_2x2.txt", "mm_2x3x2.txt"])
def test_o1_golden_hand_cases(name):
    g = load_golden(name)
    C = oracle.gemm(f32(g["A"]), f32(g["B"]))
    assert np.array_equal(C, g["C"])


def test_o1_brute_force_tiny():
    rng = np.random.default_rng(0)
    for (M, N, K) in [(1, 1, 1), (3, 4, 5), (5, 2, 7)]:
        A = f32(rng.standard_normal((M, K)))
        B = f32(rng.standard_normal((K, N)))
        ref = np.zeros((M, N))
        for i in range(M):
            for j in range(N):
                s = 0.0
                for k in range(K):
                    s += float(A[i, k]) * float(B[k, j])
                ref[i, j] = s
        C = oracle.gemm(A, B)
        assert np.allclose(C, ref, rtol=1e-15, atol=1e-15)


def test_o1_closed_forms():
    M, N, K = 33, 47, 29
    A = nugen.fill(M, K, 1, 1)
    B = nugen.fill(K, N, 1, 2)
    I_K = np.eye(K, dtype=np.float32)
    I_M = np.eye(M, dtype=np.float32)
    assert np.array_equal(oracle.gemm(A, I_K), A.astype(np.float64))      # A.I = A
    assert np.array_equal(oracle.gemm(I_M, A), A.astype(np.float64))      # I.A = A
    ones = oracle.gemm(np.ones((M, K), np.float32), np.ones((K, N), np.float32))
    assert np.array_equal(ones, np.full((M, N), float(K)))                # 1.1 = K
    # rank-1: (u v^T)(w z^T) = (v.w) u z^T with small integers
    rng = np.random.default_rng(1)
    u, v = rng.integers(-5, 6, M), rng.integers(-5, 6, K)
    w, z = rng.integers(-5, 6, K), rng.integers(-5, 6, N)
    C = oracle.gemm(f32(np.outer(u, v)), f32(np.outer(w, z)))
    assert np.array_equal(C, float(v @ w) * np.outer(u, z).astype(np.float64))
    # diagonal scaling: D B scales row k of B by d_k
    d = rng.integers(-4, 5, K).astype(np.float32)
    assert np.array_equal(oracle.gemm(np.diag(d), B), d[:, None].astype(np.float64) * B)


@pytest.mark.parametrize("shape", [(1, 1, 1), (257, 129, 65), (1, 300, 40), (64, 64, 64)])
def test_o1_matches_library_dgemm(shape):
    M, N, K = shape
    Ai = nugen.fill(M, K, 7, 1, "int")
    Bi = nugen.fill(K, N, 7, 2, "int")
    # integer inputs: every partial sum is exact in fp64 -> bitwise
    assert np.array_equal(oracle.gemm(Ai, Bi), Ai.astype(np.float64) @ Bi.astype(np.float64))
    A = nugen.fill(M, K, 7, 1)
    B = nugen.fill(K, N, 7, 2)
    ref = A.astype(np.float64) @ B.astype(np.float64)
    C = oracle.gemm(A, B)
    scale = np.abs(A).astype(np.float64) @ np.abs(B).astype(np.float64)
    assert np.all(np.abs(C - ref) <= 1e-13 * scale + 1e-300)


def test_o1_transposed_operand_is_caught():
    """A plausible mistake (using B^T) must fail the pins above."""
    A = nugen.fill(8, 8, 1, 1, "int")
    B = nugen.fill(8, 8, 1, 2, "int")
    assert not np.array_equal(oracle.gemm(A, np.ascontiguousarray(B.T)),
                              A.astype(np.float64) @ B.astype(np.float64))


def test_o1_strided_views():
    A = nugen.fill(20, 30, 3, 1, "int")
    B = nugen.fill(30, 40, 3, 2, "int")
    sub = oracle.gemm(A[2:9], B[:, 5:17].copy())
    assert np.array_equal(sub, A[2:9].astype(np.float64) @ B[:, 5:17].astype(np.float64))


def test_rows_and_entries_agree_with_full():
    A = nugen.fill(50, 70, 4, 1)
    B = nugen.fill(70, 30, 4, 2)
    C = oracle.gemm(A, B)
    rows = [0, 17, 49]
    assert np.array_equal(oracle.gemm_rows(A, B, rows), C[rows])
    I = [0, 3, 49, 10]
    J = [0, 29, 5, 10]
    e = oracle.entries(A, B, I, J)
    assert np.allclose(e, C[I, J], rtol=1e-14, atol=1e-14)


def test_norms():
    A = nugen.fill(9, 11, 5, 1)
    B = nugen.fill(11, 13, 5, 2)
    assert np.allclose(oracle.row_norms(A), np.linalg.norm(A.astype(np.float64), axis=1))
    assert np.allclose(oracle.col_norms(B), np.linalg.norm(B.astype(np.float64), axis=0))


def test_normwise_checker_flags_planted_error():
    M, N, K = 40, 30, 50
    A = nugen.fill(M, K, 6, 1)
    B = nugen.fill(K, N, 6, 2)
    R = oracle.gemm(A, B)
    rn, cn = oracle.row_norms(A), oracle.col_norms(B)
    C = R.astype(np.float32)
    e0, _ = oracle.normwise_err(C, R, rn, cn)
    assert e0 < 1e-7                              # fp32 rounding of the exact result
    bad = C.copy()
    bad[7, 11] += np.float32(2e-5 * rn[7] * cn[11])
    e1, (i, j) = oracle.normwise_err(bad, R, rn, cn)
    assert (i, j) == (7, 11) and 1.9e-5 < e1 < 2.1e-5
    nan = C.copy()
    nan[0, 0] = np.nan
    assert oracle.normwise_err(nan, R, rn, cn)[0] == np.inf


def test_freivalds_exact_on_integers_and_detects_misplaced_block():
    M, N, K = 64, 48, 80
    A = nugen.fill(M, K, 8, 1, "int")
    B = nugen.fill(K, N, 8, 2, "int")
    C = oracle.gemm(A, B).astype(np.float32)       # exact: |sums| << 2^24
    r = np.where(np.random.default_rng(0).random(N) < 0.5, -1.0, 1.0)
    e, x, y = oracle.freivalds(A, B, C, r)
    assert e == 0.0 and np.array_equal(x, y)
    bad = C.copy()
    bad[16:32, 8:16] = C[0:16, 8:16]               # a block copied to the wrong place
    e2, x2, y2 = oracle.freivalds(A, B, bad, r)
    assert not np.array_equal(x2, y2)


def test_freivalds_ratio_scale_pinned_by_planted_row_error():
    """The normalised ratio |(C r)_i - (A (B r))_i| / (||A_i|| sum_j ||B_j|| |r_j|)
    (SURVEY §8(c) "Large configs") is pinned to its closed form: a planted
    row-wide error Delta_ij = eps ||A_i|| ||B_j|| r_j (same sign as r_j, so no
    cancellation) gives (Delta r)_i = eps ||A_i|| sum_j ||B_j|| |r_j| exactly,
    i.e. a ratio of eps.  A scale bug (sum ||B_j||^2, a stray factor N, a
    missing ||A_i||) moves the ratio off eps; the fp32-rounded exact C stays far
    below TOL, and eps = 2e-5 > TOL = 1e-5 fails the check."""
    M, N, K = 48, 64, 96
    A = nugen.fill(M, K, 31, 1)
    B = nugen.fill(K, N, 31, 2)
    R = oracle.gemm(A, B)
    rn, cn = oracle.row_norms(A), oracle.col_norms(B)
    r = np.where(np.random.default_rng(5).random(N) < 0.5, -1.0, 1.0)
    C = R.astype(np.float32)
    e0, _, _ = oracle.freivalds(A, B, C, r)
    assert e0 < 1e-7                                 # fp32 rounding of the exact result
    for i, eps in ((5, 2e-5), (40, 3e-6)):
        bad = R.copy()
        bad[i, :] += eps * rn[i] * cn * r            # the planted row error, in fp64
        # compare in fp64 so the planted value is not lost to fp32 rounding
        e, x, y = oracle.freivalds(A, B, bad.astype(np.float32), r)
        dx = (bad.astype(np.float32).astype(np.float64) - R) @ r
        ratio_i = abs(dx[i]) / (rn[i] * float(np.sum(cn * np.abs(r))))
        assert abs(ratio_i - eps) < 0.05 * eps      # the closed form, through fp32 rounding
        assert abs(e - ratio_i) < 1e-7               # the oracle reports that row's ratio
        assert (e > 1e-5) == (eps > 1e-5)            # 2e-5 fails TOL, 3e-6 passes


def test_freivalds_integer_exact_detects_single_element():
    """On integer inputs x = C r and y = A (B r) are exact in fp64, so a single
    wrong element (off by 1) is detected however large N is (no dilution)."""
    M, N, K = 40, 300, 50
    A = nugen.fill(M, K, 32, 1, "int")
    B = nugen.fill(K, N, 32, 2, "int")
    C = oracle.gemm(A, B).astype(np.float32)
    r = np.where(np.random.default_rng(6).random(N) < 0.5, -1.0, 1.0)
    _, x, y = oracle.freivalds(A, B, C, r)
    assert np.array_equal(x, y)
    C[17, 222] += 1.0
    _, x2, y2 = oracle.freivalds(A, B, C, r)
    assert np.flatnonzero(x2 != y2).tolist() == [17] and abs(x2[17] - y2[17]) == 1.0


@settings(max_examples=25, deadline=None)
@given(M=st.integers(1, 40), N=st.integers(1, 40), K=st.integers(0, 40),
       bm=st.integers(1, 17), bn=st.integers(1, 17), bk=st.integers(1, 17),
       depth=st.integers(1, 3), reuse=st.booleans(), order=st.sampled_from(["mn", "nm"]))
def test_o2_recursive_equals_o1_on_integers(M, N, K, bm, bn, bk, depth, reuse, order):
    A = nugen.fill(M, K, 9, 1, "int")
    B = nugen.fill(K, N, 9, 2, "int")
    levels = [(max(1, bm >> l), max(1, bn >> l), max(1, bk >> l)) for l in range(depth)]
    C2 = oracle.recursive(A, B, levels, reuse_row_shard=reuse, order=order)
    C1 = oracle.gemm(A, B) if K > 0 else np.zeros((M, N))
    assert np.array_equal(C2, C1)


def test_o2_row_shard_reuse_invariant_on_uniform():
    A = nugen.fill(37, 53, 10, 1)
    B = nugen.fill(53, 29, 10, 2)
    lv = [(16, 8, 20), (5, 4, 7)]
    a = oracle.recursive(A, B, lv, reuse_row_shard=False)
    b = oracle.recursive(A, B, lv, reuse_row_shard=True)
    assert np.array_equal(a, b)
    C1 = oracle.gemm(A, B)
    assert np.allclose(a, C1, rtol=0, atol=1e-12)


def test_o2_detects_dropped_block():
    """A plausible decomposition mistake (dropping the ragged last k-block)
    changes the result, so the O2 == O1 pin is not vacuous."""
    A = nugen.fill(10, 10, 11, 1, "int")
    B = nugen.fill(10, 10, 11, 2, "int")
    full = oracle.recursive(A, B, [(4, 4, 4)])
    trunc = oracle.recursive(A[:, :8].copy(), B[:8].copy(), [(4, 4, 4)])
    assert not np.array_equal(full, trunc)
