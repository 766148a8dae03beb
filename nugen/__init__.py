"""nugen — seeded counter-based input generator.

Shared by the harness (bench.py, tests) and by the oracle's checks. It holds
none of the GEMM method's arithmetic: it maps a global coordinate (i, j) of
matrix `mat` to a value, so a sub-block can be regenerated anywhere.

Three implementations of the same recipe, cross-checked in tests/test_gen.py:
  * `fill`        — the C/OpenMP library (libnugen.so) used for large inputs;
  * `fill_numpy`  — vectorised numpy uint64 arithmetic;
  * `entry_py`    — pure Python integers (the brute-force definition).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

UNIFORM, INT, EYE, ONES, RANK1, ZEROS, TEMP, POWER = 0, 1, 2, 3, 4, 5, 6, 7
KINDS = {"uniform": UNIFORM, "int": INT, "eye": EYE, "ones": ONES,
         "rank1": RANK1, "zeros": ZEROS, "temp": TEMP, "power": POWER}
MAT_A, MAT_B = 1, 2
MAT_T, MAT_P = 3, 4      # HotSpot-2D temperature and power grids (NEXT-3)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libnugen.so")
_lib = None

_M64 = (1 << 64) - 1
_GOLDEN = 0x9E3779B97F4A7C15


def build(force: bool = False) -> str:
    """Compile libnugen.so with gcc -O3 -fopenmp (idempotent)."""
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v3", "-fopenmp", "-shared",
                               "-fPIC", "-o", _SO, src])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        lib.nugen_fill_f32.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64,
                                       ctypes.c_int, ctypes.c_int, ctypes.c_int64,
                                       ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                                       ctypes.c_int64]
        lib.nugen_fill_f32.restype = None
        lib.nugen_entry.argtypes = [ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
                                    ctypes.c_int64, ctypes.c_int64, ctypes.c_int64]
        lib.nugen_entry.restype = ctypes.c_float
        _lib = lib
    return _lib


def _kind(kind) -> int:
    return KINDS[kind] if isinstance(kind, str) else int(kind)


def fill_ptr(ptr: int, ld: int, seed: int, mat: int, kind, ncols: int,
             i0: int, j0: int, rows: int, cols: int) -> None:
    """Fill rows x cols fp32 values at raw host address `ptr` (row-major, ld)."""
    if rows <= 0 or cols <= 0:
        return
    _load().nugen_fill_f32(ctypes.c_void_p(ptr), ld, seed & _M64, mat, _kind(kind),
                           ncols, i0, j0, rows, cols)


def fill(rows: int, cols: int, seed: int, mat: int, kind="uniform", out=None,
         i0: int = 0, j0: int = 0, ncols: int | None = None) -> np.ndarray:
    """Return (or fill `out` with) the rows x cols block at (i0, j0) of a
    matrix with `ncols` columns (default: cols)."""
    ncols = cols if ncols is None else ncols
    if out is None:
        out = np.empty((rows, cols), dtype=np.float32)
    if rows <= 0 or cols <= 0:
        return out
    assert out.dtype == np.float32 and out.ndim == 2 and out.strides[1] == 4
    fill_ptr(out.ctypes.data, out.strides[0] // 4, seed, mat, kind, ncols, i0, j0,
             rows, cols)
    return out


def _splitmix64_np(z: np.ndarray) -> np.ndarray:
    z = z + np.uint64(_GOLDEN)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def fill_numpy(rows: int, cols: int, seed: int, mat: int, kind="uniform",
               i0: int = 0, j0: int = 0, ncols: int | None = None) -> np.ndarray:
    """Vectorised numpy version of the same recipe (independent of the C code)."""
    k = _kind(kind)
    ncols = cols if ncols is None else ncols
    i = np.arange(i0, i0 + rows, dtype=np.uint64)[:, None]
    j = np.arange(j0, j0 + cols, dtype=np.uint64)[None, :]
    with np.errstate(over="ignore"):
        base = np.uint64((seed * _GOLDEN) & _M64) ^ np.uint64((mat << 56) & _M64)
        if k in (UNIFORM, INT, TEMP, POWER):
            h = _splitmix64_np(base ^ (i * np.uint64(ncols) + j))
            if k in (UNIFORM, TEMP, POWER):
                q = (h >> np.uint64(40)).astype(np.int64) - (1 << 23)
                u = q.astype(np.float64) * 2.0 ** -23
                if k == TEMP:
                    return (330.0 + 10.0 * u).astype(np.float32)
                if k == POWER:
                    return (0.25 + 0.25 * u).astype(np.float32)
                return u.astype(np.float32)
            return ((h % np.uint64(17)).astype(np.int64) - 8).astype(np.float32)
        if k == EYE:
            return (i == j).astype(np.float32)
        if k == ONES:
            return np.ones((rows, cols), dtype=np.float32)
        if k == RANK1:
            hu = _splitmix64_np(base ^ (i ^ np.uint64(0x0F0F0F0F0F0F)))
            basev = np.uint64((seed * _GOLDEN) & _M64) ^ np.uint64(((mat ^ 0x40) << 56) & _M64)
            hv = _splitmix64_np(basev ^ (j ^ np.uint64(0x0F0F0F0F0F0F)))
            u = (hu & np.uint64(7)).astype(np.int64) - 3
            v = (hv & np.uint64(7)).astype(np.int64) - 3
            return (u * v).astype(np.float32)
        return np.zeros((rows, cols), dtype=np.float32)


def _splitmix64_py(z: int) -> int:
    z = (z + _GOLDEN) & _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def entry_py(seed: int, mat: int, kind, ncols: int, i: int, j: int) -> float:
    """Pure-Python definition of one entry (brute force, for pinning)."""
    k = _kind(kind)
    base = ((seed * _GOLDEN) & _M64) ^ ((mat << 56) & _M64)
    if k in (UNIFORM, TEMP, POWER):
        h = _splitmix64_py(base ^ ((i * ncols + j) & _M64))
        u = float(((h >> 40) - (1 << 23)) * 2.0 ** -23)
        if k == TEMP:
            return float(np.float32(330.0 + 10.0 * u))
        if k == POWER:
            return float(np.float32(0.25 + 0.25 * u))
        return u
    if k == INT:
        h = _splitmix64_py(base ^ ((i * ncols + j) & _M64))
        return float(h % 17 - 8)
    if k == EYE:
        return 1.0 if i == j else 0.0
    if k == ONES:
        return 1.0
    if k == RANK1:
        hu = _splitmix64_py(base ^ (i ^ 0x0F0F0F0F0F0F))
        basev = ((seed * _GOLDEN) & _M64) ^ (((mat ^ 0x40) << 56) & _M64)
        hv = _splitmix64_py(basev ^ (j ^ 0x0F0F0F0F0F0F))
        return float(((hu & 7) - 3) * ((hv & 7) - 3))
    return 0.0


def entry(seed: int, mat: int, kind, ncols: int, i: int, j: int) -> float:
    return float(_load().nugen_entry(seed & _M64, mat, _kind(kind), ncols, i, j))
