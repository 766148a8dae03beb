"""Parity of the sm_100a leaf (scaled fp16 hi/lo split, three tcgen05 MMAs per
16 k; R22) with the fp64 oracle, called through the C ABI
(northup_leaf_gemm) on device memory, and through northup_gemm on a HOST ->
HBM tree for the adversarial cases.

Bar (BASELINE.json north_star): max |C - C_ref| / (||A_i,:||_2 ||B_:,j||_2)
<= 1e-5; integer inputs in [-8, 8] split exactly (hi = x, lo = 0) and every
partial sum is exact in fp32, so those must match the oracle bit for bit
(SURVEY.md §8(c))."""
import numpy as np
import pytest
import torch

import nugen
import oracle
import paper_conf_ipps_chey19_b200 as nu

pytestmark = pytest.mark.gpu
TOL = 1e-5


def _dev():
    assert torch.cuda.is_available(), "GPU tests need a B200"
    return torch.device("cuda:0")


def run_leaf(A, B, C0=None, accumulate=False, k_chunk=0, npass=0, lda_pad=0, ldb_pad=0, ldc_pad=0):
    dev = _dev()
    M, K = A.shape
    N = B.shape[1]
    r4 = lambda x: -(-x // 4) * 4                      # TMA: 16-byte row pitch
    Ad = torch.zeros((M, r4(K) + lda_pad), dtype=torch.float32, device=dev)
    Bd = torch.zeros((K, r4(N) + ldb_pad), dtype=torch.float32, device=dev)
    Cd = torch.full((M, N + ldc_pad), float("nan"), dtype=torch.float32, device=dev)
    Ad[:, :K] = torch.from_numpy(A)
    Bd[:, :N] = torch.from_numpy(B)
    if C0 is not None:
        Cd[:, :N] = torch.from_numpy(C0)
    nu.leaf_gemm(Ad[:, :K], Bd[:, :N], Cd[:, :N], accumulate=accumulate, k_chunk=k_chunk,
                 npass=npass)
    torch.cuda.synchronize()
    out = Cd.cpu().numpy()
    if ldc_pad:
        assert np.isnan(out[:, N:]).all(), "kernel wrote outside its C columns"
    return np.ascontiguousarray(out[:, :N])


def normwise(C, A, B, ref=None):
    ref = oracle.gemm(A, B) if ref is None else ref
    return oracle.normwise_err(C, ref, oracle.row_norms(A), oracle.col_norms(B))[0]


SHAPES = [(128, 256, 32), (256, 512, 64), (257, 300, 65), (1, 1, 1), (64, 64, 64), (33, 17, 40),
          (130, 260, 100), (512, 256, 1024), (384, 768, 2056), (1000, 1000, 999)]


@pytest.mark.parametrize("M,N,K", SHAPES)
def test_leaf_integer_inputs_bitwise(M, N, K):
    A = nugen.fill(M, K, 11, 1, "int")
    B = nugen.fill(K, N, 11, 2, "int")
    C = run_leaf(A, B)
    ref = oracle.gemm(A, B)
    assert np.array_equal(C.astype(np.float64), ref), \
        f"{np.argwhere(C.astype(np.float64) != ref)[:5]}"


@pytest.mark.parametrize("npass", [3, 4])
@pytest.mark.parametrize("M,N,K", SHAPES)
def test_leaf_uniform_normwise(M, N, K, npass):
    A = nugen.fill(M, K, 12, 1)
    B = nugen.fill(K, N, 12, 2)
    C = run_leaf(A, B, npass=npass)
    e = normwise(C, A, B)
    assert e <= TOL, e


@pytest.mark.parametrize("M,N,K", [(257, 300, 65), (512, 256, 1024), (1000, 1000, 999)])
def test_leaf_npass4_integer_bitwise(M, N, K):
    A = nugen.fill(M, K, 11, 1, "int")
    B = nugen.fill(K, N, 11, 2, "int")
    assert np.array_equal(run_leaf(A, B, npass=4).astype(np.float64), oracle.gemm(A, B))


def test_leaf_closed_forms():
    M, N, K = 300, 260, 520
    ones = run_leaf(np.ones((M, K), np.float32), np.ones((K, N), np.float32))
    assert (ones == K).all()                                   # 1.1 = K exactly
    A = nugen.fill(M, K, 13, 1)
    I = np.eye(K, N, dtype=np.float32)
    C = run_leaf(A, I)
    assert normwise(C, A, I) <= TOL                            # A.I = A within the bound
    u = nugen.fill(M, 1, 13, 3, "int")
    v = nugen.fill(1, K, 13, 4, "int")
    w = nugen.fill(K, 1, 13, 5, "int")
    z = nugen.fill(1, N, 13, 6, "int")
    R = run_leaf(u @ v, w @ z)                                 # rank-1: (v.w) u z^T
    assert np.array_equal(R.astype(np.float64), float((v @ w)[0, 0]) * (u @ z).astype(np.float64))


def test_leaf_accumulate_and_chunks():
    M, N, K = 300, 520, 3000
    A = nugen.fill(M, K, 14, 1)
    B = nugen.fill(K, N, 14, 2)
    C0 = nugen.fill(M, N, 14, 3)
    C = run_leaf(A, B, C0=C0, accumulate=True, k_chunk=256)
    ref = oracle.gemm(A, B) + C0.astype(np.float64)
    assert normwise(C, A, B, ref=ref) <= TOL
    # K panels of 128 vs one default panel: integer inputs identical
    Ai = nugen.fill(M, K, 15, 1, "int")
    Bi = nugen.fill(K, N, 15, 2, "int")
    assert np.array_equal(run_leaf(Ai, Bi, k_chunk=128), run_leaf(Ai, Bi, k_chunk=0))


def test_leaf_strided_unaligned_operands_and_predicated_stores():
    """Any leading dimension (the split reads A and B with plain loads): odd lda
    / ldb, 4-byte-offset bases, ldc % 4 != 0 (register epilogue, not TMA)."""
    M, N, K = 200, 130, 96
    A = nugen.fill(M, K, 16, 1, "int")
    B = nugen.fill(K, N, 16, 2, "int")
    C = run_leaf(A, B, lda_pad=36, ldb_pad=12, ldc_pad=5)
    assert np.array_equal(C.astype(np.float64), oracle.gemm(A, B))
    dev = _dev()
    Ad = torch.zeros((M, K + 3), device=dev)
    Ad[:, 1:K + 1] = torch.from_numpy(A)
    Bd = torch.zeros((K, N + 1), device=dev)
    Bd[:, :N] = torch.from_numpy(B)
    Cd = torch.full((M, N + 3), float("nan"), device=dev)
    nu.leaf_gemm(Ad[:, 1:K + 1], Bd[:, :N], Cd[:, 1:N + 1])
    torch.cuda.synchronize()
    out = Cd.cpu().numpy()
    assert np.array_equal(out[:, 1:N + 1].astype(np.float64), oracle.gemm(A, B))
    assert np.isnan(out[:, 0]).all() and np.isnan(out[:, N + 1:]).all()


def test_leaf_hi_only_fails_the_bound():
    """Reading R9/R22 negative test: the hi.hi product alone (npass = 1, fp16
    with 11 significant bits) must NOT meet 1e-5 - the cross terms are what
    buys fp32-level accuracy."""
    A = nugen.fill(256, 512, 17, 1)
    B = nugen.fill(512, 256, 17, 2)
    e1 = normwise(run_leaf(A, B, npass=1), A, B)
    e3 = normwise(run_leaf(A, B, npass=3), A, B)
    e4 = normwise(run_leaf(A, B, npass=4), A, B)
    assert e1 > 1e-5 > TOL / 4 > max(e3, e4)


def test_leaf_rejects_unknown_npass():
    dev = _dev()
    A = torch.zeros((8, 8), device=dev)
    with pytest.raises(nu.NorthupError) as e:
        nu.leaf_gemm(A, A, torch.zeros((8, 8), device=dev), npass=2)
    assert e.value.code == nu.NU_EINVAL


def test_leaf_degenerate_sizes():
    dev = _dev()
    C = torch.full((5, 6), 3.0, device=dev)
    nu.leaf_gemm(torch.zeros((5, 0), device=dev), torch.zeros((0, 6), device=dev), C)
    torch.cuda.synchronize()
    assert (C == 0).all()             # K = 0: C = A.B = 0
    C2 = torch.full((5, 6), 3.0, device=dev)
    nu.leaf_gemm(torch.zeros((5, 0), device=dev), torch.zeros((0, 6), device=dev), C2,
                 accumulate=True)
    torch.cuda.synchronize()
    assert (C2 == 3).all()            # K = 0 with accumulate: untouched


def test_leaf_integer_exact_and_clipped_edges():
    """Integer inputs over several K panels: exact vs the oracle; C columns
    beyond N (ldc > N) and rows beyond M stay untouched by the TMA epilogue."""
    dev = _dev()
    M, N, K = 261, 300, 4100
    A = nugen.fill(M, K, 21, 1, "int")
    B = nugen.fill(K, N, 21, 2, "int")
    Ad = torch.from_numpy(A).to(dev)
    Bd = torch.from_numpy(B).to(dev)
    big = torch.full((M + 3, 308), float("nan"), device=dev)
    nu.leaf_gemm(Ad, Bd, big[:M, :N])
    torch.cuda.synchronize()
    out = big.cpu().numpy()
    assert np.array_equal(out[:M, :N].astype(np.float64), oracle.gemm(A, B))
    assert np.isnan(out[:M, N:]).all() and np.isnan(out[M:]).all()


def test_leaf_wide_n_is_split_in_column_pieces():
    """N above the leaf's B split width (32768 columns) runs in column pieces
    that reuse A's split: exact on integers."""
    M, N, K = 64, 40000, 96
    A = nugen.fill(M, K, 23, 1, "int")
    B = nugen.fill(K, N, 23, 2, "int")
    assert np.array_equal(run_leaf(A, B).astype(np.float64), oracle.gemm(A, B))


def test_leaf_deterministic():
    A = nugen.fill(700, 1500, 22, 1)
    B = nugen.fill(1500, 900, 22, 2)
    assert np.array_equal(run_leaf(A, B), run_leaf(A, B))


def test_leaf_scale_exponent_edges():
    """Rows / columns that are all zero, or far from 1 (1e-20 .. 1e20), get their
    own power-of-two exponents (R22): the bound holds row by row.  (Products
    stay inside fp32's normal range - reading R17: results that underflow or
    overflow fp32 are out of scope for any fp32 implementation.)"""
    M, N, K = 96, 80, 640
    A = nugen.fill(M, K, 24, 1)
    B = nugen.fill(K, N, 24, 2)
    A[3] = 0.0
    A[5] *= np.float32(1e-20)
    A[7] *= np.float32(1e20)
    B[:, 2] = 0.0
    B[:, 9] *= np.float32(1e-15)
    B[:, 11] *= np.float32(1e15)
    C = run_leaf(A, B)
    assert (C[3] == 0).all() and (C[:, 2] == 0).all()
    assert normwise(C, A, B) <= TOL


# ------------------------------------------------ adversarial inputs
# Same-sign data: every product's split error and every accumulator truncation
# (the tensor core truncates its fp32 accumulator after each MMA, R20) push the
# sum the same way, so nothing cancels.  A = B = c.1 makes the normwise error
# equal the relative error of one dot product.
ADV_CONST = [1.0048771, 0.3, 0.1256096, 1.0 - 2.0 ** -12]


def _adv_inputs(kind, M, N, K):
    if kind.startswith("const"):
        c = np.float32(float(kind[5:]))
        return np.full((M, K), c, np.float32), np.full((K, N), c, np.float32)
    rng = np.random.default_rng(K)
    if kind == "u01":
        return rng.random((M, K), dtype=np.float32), rng.random((K, N), dtype=np.float32)
    if kind == "scaled":   # rows of A over 2^-40..2^40, columns of B over 2^30..2^-30
        A = (rng.random((M, K), dtype=np.float32) * 2 - 1) * np.exp2(np.linspace(-40, 40, M))[:, None]
        B = (rng.random((K, N), dtype=np.float32) * 2 - 1) * np.exp2(np.linspace(30, -30, N))[None, :]
        return A.astype(np.float32), B.astype(np.float32)
    raise ValueError(kind)


ADV_KINDS = [f"const{c!r}" for c in ADV_CONST] + ["u01", "scaled"]


@pytest.mark.parametrize("K", [2048, 32768])
@pytest.mark.parametrize("kind", ADV_KINDS)
def test_leaf_adversarial_direct(kind, K):
    M = N = 256
    A, B = _adv_inputs(kind, M, N, K)
    e = normwise(run_leaf(A, B), A, B)
    assert e <= TOL / 2, e      # R22 budget: split <= 7.2e-7 per product + measured accumulation <= 3.1e-6


@pytest.mark.parametrize("K", [2048, 32768])
@pytest.mark.parametrize("kind", ["const1.0048771", "const0.3", "u01"])
def test_leaf_adversarial_through_tree(kind, K):
    """The same inputs through northup_gemm: pinned HOST root -> HBM (capped so
    K streams in panels) -> SMEM/TMEM leaf."""
    import ctypes
    M, N = 256, 384
    A, B = _adv_inputs(kind, M, N, K)
    t, _ = nu.host_tree(1, 64 << 20)
    t.finalize()
    bA, bB, bC = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
    view = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
    view(bA, M, K)[:] = A
    view(bB, K, N)[:] = B
    st = t.gemm(bA, bB, bC, M, N, K)
    C = view(bC, M, N).copy()
    t.destroy()
    assert st["bytes_h2d"] >= 4 * (M * K + K * N)
    assert normwise(C, A, B) <= TOL / 2


def test_leaf_small_panel_fused_split_matches_regular_split():
    """Small panels (A and B together <= 2^21 elements) take the one-launch
    fused split; the split is per row of A and per column of B, so a small
    sub-problem reproduces the matching block of a large (regular-split)
    product bit for bit."""
    M, N, K = 2048, 1536, 1024
    A = nugen.fill(M, K, 27, 1)
    B = nugen.fill(K, N, 27, 2)
    big = run_leaf(A, B)
    small = run_leaf(np.ascontiguousarray(A[:64]), np.ascontiguousarray(B[:, :512]))
    assert np.array_equal(small, big[:64, :512])
    assert normwise(small, A[:64], B[:, :512]) <= TOL
