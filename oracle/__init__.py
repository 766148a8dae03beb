"""ORACLE — TEST INFRASTRUCTURE ONLY.

Plain fp64 CPU reference for the Northup dense matrix multiply (PAPER.md
§IV-A).  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / `--impl reference` leg may import this package.  It shares no
code with the CUDA path (paper_conf_ipps_chey19_b200/) and never imports it.

  * O1 `gemm`        — the definition C_ref[i,j] = sum_k A[i,k] B[k,j] in fp64
                       (oracle.c, plain i-k-j triple loop, OpenMP over rows);
  * O2 `recursive`   — Listing 3 / §IV-A literally: row and column shards are
                       copied down a level, partial products accumulated,
                       C blocks copied up (recursive.py);
  * checks           — row/column norms, the normwise error of BASELINE.json
                       (max |C - C_ref| / (||A_i,:||_2 ||B_:,j||_2)), sampled
                       entries and Freivalds' check for full-size configs.
  * `oracle.hotspot` — HotSpot-2D, the paper's stencil case study (§IV-B,
                       P:307-325; S§8(f) NEXT-3): the update, [18]'s explicit
                       edge cases, the blocked recursion, the fp32 bound.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .recursive import recursive  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

_f = ctypes.c_void_p
_i64 = ctypes.c_int64


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc -O3 -fopenmp, no FMA contraction)."""
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v3", "-ffp-contract=off",
                               "-fopenmp", "-shared", "-fPIC", "-o", _SO, src, "-lm"])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        lib.oracle_gemm.argtypes = [_f, _i64, _f, _i64, _f, _i64, _i64, _i64, _i64]
        lib.oracle_gemm.restype = None
        lib.oracle_gemm_rows.argtypes = [_f, _i64, _f, _i64, _f, _i64, _f, _i64, _i64, _i64]
        lib.oracle_gemm_rows.restype = None
        lib.oracle_entries.argtypes = [_f, _i64, _f, _i64, _i64, _f, _f, _i64, _f]
        lib.oracle_entries.restype = None
        lib.oracle_row_norms.argtypes = [_f, _i64, _i64, _i64, _f]
        lib.oracle_row_norms.restype = None
        lib.oracle_col_norms.argtypes = [_f, _i64, _i64, _i64, _f]
        lib.oracle_col_norms.restype = None
        lib.oracle_normwise_err.argtypes = [_f, _i64, _f, _i64, _f, _f, _i64, _i64, _f, _f]
        lib.oracle_normwise_err.restype = ctypes.c_double
        lib.oracle_freivalds.argtypes = [_f, _i64, _f, _i64, _f, _i64, _i64, _i64, _i64,
                                         _f, _f, _f, _f, _f]
        lib.oracle_freivalds.restype = ctypes.c_double
        lib.oracle_threads.argtypes = []
        lib.oracle_threads.restype = ctypes.c_int
        lib.oracle_set_threads.argtypes = [ctypes.c_int]
        lib.oracle_set_threads.restype = None
        _lib = lib
    return _lib


def threads() -> int:
    return int(_load().oracle_threads())


def set_threads(n: int) -> None:
    _load().oracle_set_threads(int(n))


def _f32(x: np.ndarray) -> np.ndarray:
    assert x.dtype == np.float32 and x.ndim == 2, "2-D fp32"
    if x.size and x.strides[1] != 4:
        raise ValueError("row-major fp32 with unit column stride required")
    return x


def _ld(x: np.ndarray) -> int:
    return x.strides[0] // x.itemsize


def gemm(A: np.ndarray, B: np.ndarray) -> np.ndarray:
    """O1: C_ref = A B in fp64, A (M x K), B (K x N) fp32."""
    A, B = _f32(A), _f32(B)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    C = np.zeros((M, N), dtype=np.float64)
    if M and N:
        _load().oracle_gemm(A.ctypes.data, _ld(A), B.ctypes.data, _ld(B), C.ctypes.data,
                            N, M, N, K)
    return C


def gemm_rows(A: np.ndarray, B: np.ndarray, rows) -> np.ndarray:
    A, B = _f32(A), _f32(B)
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    N = B.shape[1]
    out = np.empty((len(rows), N), dtype=np.float64)
    if len(rows) and N:
        _load().oracle_gemm_rows(A.ctypes.data, _ld(A), B.ctypes.data, _ld(B),
                                 rows.ctypes.data, len(rows), out.ctypes.data, N, N,
                                 A.shape[1])
    return out


def entries(A: np.ndarray, B: np.ndarray, I, J) -> np.ndarray:
    A, B = _f32(A), _f32(B)
    I = np.ascontiguousarray(I, dtype=np.int64)
    J = np.ascontiguousarray(J, dtype=np.int64)
    out = np.empty(len(I), dtype=np.float64)
    if len(I):
        _load().oracle_entries(A.ctypes.data, _ld(A), B.ctypes.data, _ld(B), A.shape[1],
                               I.ctypes.data, J.ctypes.data, len(I), out.ctypes.data)
    return out


def row_norms(A: np.ndarray) -> np.ndarray:
    A = _f32(A)
    out = np.empty(A.shape[0], dtype=np.float64)
    if A.shape[0]:
        _load().oracle_row_norms(A.ctypes.data, _ld(A), A.shape[0], A.shape[1],
                                 out.ctypes.data)
    return out


def col_norms(B: np.ndarray) -> np.ndarray:
    B = _f32(B)
    out = np.empty(B.shape[1], dtype=np.float64)
    if B.shape[1]:
        _load().oracle_col_norms(B.ctypes.data, _ld(B), B.shape[0], B.shape[1],
                                 out.ctypes.data)
    return out


def normwise_err(C: np.ndarray, Cref: np.ndarray, rn: np.ndarray, cn: np.ndarray):
    """max |C - C_ref| / (||A_i||_2 ||B_j||_2) and its (i, j) (BASELINE.json)."""
    C = _f32(C)
    Cref = np.ascontiguousarray(Cref, dtype=np.float64)
    rn = np.ascontiguousarray(rn, dtype=np.float64)
    cn = np.ascontiguousarray(cn, dtype=np.float64)
    M, N = Cref.shape
    if M == 0 or N == 0:
        return 0.0, (-1, -1)
    ai, aj = ctypes.c_int64(), ctypes.c_int64()
    e = _load().oracle_normwise_err(C.ctypes.data, _ld(C), Cref.ctypes.data, N,
                                    rn.ctypes.data, cn.ctypes.data, M, N,
                                    ctypes.addressof(ai), ctypes.addressof(aj))
    return float(e), (ai.value, aj.value)


def freivalds(A: np.ndarray, B: np.ndarray, C: np.ndarray, r: np.ndarray,
              rn: np.ndarray | None = None, cn: np.ndarray | None = None):
    """Freivalds' check with vector r: returns (max ratio, x = C r, y = A (B r))."""
    A, B, C = _f32(A), _f32(B), _f32(C)
    M, K = A.shape
    N = B.shape[1]
    r = np.ascontiguousarray(r, dtype=np.float64)
    rn = row_norms(A) if rn is None else np.ascontiguousarray(rn, dtype=np.float64)
    cn = col_norms(B) if cn is None else np.ascontiguousarray(cn, dtype=np.float64)
    x = np.empty(M, dtype=np.float64)
    y = np.empty(M, dtype=np.float64)
    e = _load().oracle_freivalds(A.ctypes.data, _ld(A), B.ctypes.data, _ld(B),
                                 C.ctypes.data, _ld(C), M, N, K, r.ctypes.data,
                                 rn.ctypes.data, cn.ctypes.data, x.ctypes.data,
                                 y.ctypes.data)
    return float(e), x, y
