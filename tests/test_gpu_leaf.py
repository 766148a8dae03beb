"""Parity of the sm_100a leaf kernel (3xTF32 tcgen05) with the fp64 oracle,
called through the C ABI (northup_leaf_gemm) on device memory.

Bar (BASELINE.json north_star): max |C - C_ref| / (||A_i,:||_2 ||B_:,j||_2)
<= 1e-5; integer inputs in [-8, 8] are exact in TF32 and every partial sum is
exact in fp32, so those must match the oracle bit for bit."""
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


@pytest.mark.parametrize("npass", [2, 3])
@pytest.mark.parametrize("M,N,K", SHAPES)
def test_leaf_uniform_normwise(M, N, K, npass):
    A = nugen.fill(M, K, 12, 1)
    B = nugen.fill(K, N, 12, 2)
    C = run_leaf(A, B, npass=npass)
    e = normwise(C, A, B)
    assert e <= TOL, e


@pytest.mark.parametrize("M,N,K", [(257, 300, 65), (512, 256, 1024), (1000, 1000, 999)])
def test_leaf_3xtf32_integer_bitwise(M, N, K):
    A = nugen.fill(M, K, 11, 1, "int")
    B = nugen.fill(K, N, 11, 2, "int")
    assert np.array_equal(run_leaf(A, B, npass=3).astype(np.float64), oracle.gemm(A, B))


def test_leaf_v0_one_cta_kernel():
    """The 1-CTA v0 kernel (kept for comparison) still meets the bar."""
    import ctypes
    f = nu.lib().northup_debug_leaf_gemm
    f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                  ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                  ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                  ctypes.c_void_p]
    M, N, K = 300, 520, 1000
    A = nugen.fill(M, K, 18, 1)
    B = nugen.fill(K, N, 18, 2)
    dev = _dev()
    Ad, Bd = torch.from_numpy(A).to(dev), torch.from_numpy(B).to(dev)
    Cd = torch.empty((M, N), device=dev)
    assert f(Ad.data_ptr(), K, Bd.data_ptr(), N, Cd.data_ptr(), N, M, N, K, 0, 0, 3, 0, None, 1,
             None) == 0
    torch.cuda.synchronize()
    assert normwise(Cd.cpu().numpy(), A, B) <= TOL


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
    # chunked vs unchunked: both within the bound; integer inputs identical
    Ai = nugen.fill(M, K, 15, 1, "int")
    Bi = nugen.fill(K, N, 15, 2, "int")
    assert np.array_equal(run_leaf(Ai, Bi, k_chunk=128), run_leaf(Ai, Bi, k_chunk=0))


def test_leaf_strided_operands_and_predicated_stores():
    M, N, K = 200, 130, 96
    A = nugen.fill(M, K, 16, 1, "int")
    B = nugen.fill(K, N, 16, 2, "int")
    C = run_leaf(A, B, lda_pad=36, ldb_pad=12, ldc_pad=5)     # ldc % 4 != 0 -> scalar path
    assert np.array_equal(C.astype(np.float64), oracle.gemm(A, B))


def test_leaf_plain_tf32_fails_the_bound():
    """Reading R9: one TF32 pass (npass=1) must NOT meet 1e-5 — the split
    (3xTF32, or tf32 hi.hi + bf16 cross terms) is what buys fp32-level
    accuracy (negative test)."""
    A = nugen.fill(256, 512, 17, 1)
    B = nugen.fill(512, 256, 17, 2)
    e1 = normwise(run_leaf(A, B, npass=1), A, B)
    e2 = normwise(run_leaf(A, B, npass=2), A, B)
    e3 = normwise(run_leaf(A, B, npass=3), A, B)
    assert e1 > 1e-4 > TOL >= max(e2, e3)


def test_leaf_rejects_tma_illegal_operands():
    dev = _dev()
    A = torch.zeros((8, 7), device=dev)
    B = torch.zeros((7, 8), device=dev)
    C = torch.zeros((8, 8), device=dev)
    with pytest.raises(nu.NorthupError) as e:
        nu.leaf_gemm(A, B, C)          # lda = 7 is not a multiple of 4
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


def test_leaf_v2_ldg_variant_parity():
    """The experimental LDG-fed pair kernel (v2, NORTHUP_LEAF=3) computes the
    same result as the default TMA-fed kernel, bit for bit."""
    import ctypes
    f = nu.lib().northup_debug_leaf_gemm
    f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                  ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                  ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                  ctypes.c_void_p]
    dev = _dev()
    for (M, N, K) in [(300, 520, 1000), (257, 132, 37 * 4)]:
        A = nugen.fill(M, K, 19, 1)
        B = nugen.fill(K, N, 19, 2)
        Ad, Bd = torch.from_numpy(A).to(dev), torch.from_numpy(B).to(dev)
        outs = []
        for variant in (2, 3):
            Cd = torch.full((M, N), float("nan"), device=dev)
            assert f(Ad.data_ptr(), K, Bd.data_ptr(), N, Cd.data_ptr(), N, M, N, K, 0, 0, 2, 0, None,
                     variant, None) == 0
            torch.cuda.synchronize()
            outs.append(Cd.cpu().numpy())
        assert np.array_equal(outs[0], outs[1])
        assert normwise(outs[0], A, B) <= TOL


def _debug_leaf(Ad, Bd, Cd, M, N, K, variant, accumulate=0, kc=0, npass=2):
    import ctypes
    f = nu.lib().northup_debug_leaf_gemm
    f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                  ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                  ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                  ctypes.c_void_p]
    rc = f(Ad.data_ptr(), Ad.stride(0), Bd.data_ptr(), Bd.stride(0), Cd.data_ptr(), Cd.stride(0),
           M, N, K, accumulate, kc, npass, 0, None, variant, None)
    assert rc == 0
    torch.cuda.synchronize()


@pytest.mark.parametrize("M,N,K,kc", [(300, 520, 1000, 0), (257, 132, 148, 0), (512, 512, 4096, 1024),
                                      (1, 4, 8, 0), (1000, 1000, 996, 256), (2048, 2304, 2048, 0)])
def test_leaf_v3_tmem_variant_parity(M, N, K, kc):
    """v3 (A' operand in TMEM, TMA store / reduce-add epilogue, NORTHUP_LEAF=4)
    computes the same products in the same order as v1.2: bitwise equal, on
    C = A.B and on C += A.B over several K panels."""
    dev = _dev()
    A = nugen.fill(M, K, 20, 1)
    B = nugen.fill(K, N, 20, 2)
    C0 = torch.from_numpy(nugen.fill(M, N, 20, 3)).to(dev)
    Ad, Bd = torch.from_numpy(A).to(dev), torch.from_numpy(B).to(dev)
    for acc in (0, 1):
        outs = []
        for variant in (2, 4):
            Cd = C0.clone() if acc else torch.full((M, N), float("nan"), device=dev)
            _debug_leaf(Ad, Bd, Cd, M, N, K, variant, accumulate=acc, kc=kc)
            outs.append(Cd.cpu().numpy())
        assert np.array_equal(outs[0], outs[1]), (acc, np.argwhere(outs[0] != outs[1])[:5])
    ref = oracle.gemm(A, B) + C0.cpu().numpy().astype(np.float64)
    assert normwise(outs[1], A, B, ref=ref) <= TOL


def test_leaf_v3_integer_exact_and_clipped_edges():
    """Integer inputs: exact vs the oracle; C columns beyond N (ldc > N) and
    rows beyond M stay untouched by the TMA-store epilogue."""
    dev = _dev()
    M, N, K = 261, 300, 2100
    A = nugen.fill(M, K, 21, 1, "int")
    B = nugen.fill(K, N, 21, 2, "int")
    Ad = torch.zeros((M, 2104), device=dev)
    Ad[:, :K] = torch.from_numpy(A)
    Bd = torch.from_numpy(B).to(dev)
    big = torch.full((M + 3, 308), float("nan"), device=dev)
    _debug_leaf(Ad[:, :K], Bd, big[:M, :N], M, N, K, 4)
    out = big.cpu().numpy()
    assert np.array_equal(out[:M, :N].astype(np.float64), oracle.gemm(A, B))
    assert np.isnan(out[:M, N:]).all() and np.isnan(out[M:]).all()
