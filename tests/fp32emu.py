"""Test-side exact fp32 emulation of the HotSpot-2D leaf's fixed update
sequence (hotspot.cu, RH4), used for bit-for-bit checks of the GPU
results.  Independent of the CUDA code; not the oracle (oracle/hotspot.py is
fp64)."""
import numpy as np

import paper_conf_ipps_chey19_b200 as nu


def fma32(a, b, c):
    """Exact fp32 fused multiply-add on arrays: the float32 product is exact in
    float64; TwoSum gives the exact error of the float64 sum; rounding that sum
    to odd and then to float32 gives the correctly rounded result (53 >= 24 + 2)."""
    p = a.astype(np.float64) * b.astype(np.float64)
    c = np.broadcast_to(np.asarray(c, dtype=np.float64), p.shape)
    s = p + c
    bb = s - p
    e = (p - (s - bb)) + (c - bb)
    even = (s.view(np.int64) & 1) == 0
    s = np.where((e != 0) & even, np.nextafter(s, np.where(e > 0, np.inf, -np.inf)), s)
    return s.astype(np.float32)


def emulate_fp32(T, P, iters, k=None):
    """The update in fp32 in the kernel's fixed sequence (RH4, the
    expanded form; test-side check, independent of the CUDA code):
        kt = 1 - cap (2 rx + 2 ry + rz), kx = cap rx, ky = cap ry, kq = cap rz amb
        (each computed in float64 from the fp32 coefficients, rounded once)
        q = fma(cap, p, kq)                                   once per cell
        u = fma(kt, t, q); u = fma(kx, e + w, u); t' = fma(ky, s + n, u)"""
    k = nu.hotspot_coeffs(*T.shape) if k is None else k
    f = np.float32
    cap, rx, ry, rz, amb = (float(f(x)) for x in (k.cap_1, k.rx_1, k.ry_1, k.rz_1, k.amb))
    kt = np.full(T.shape, f(1.0 - cap * (2.0 * rx + 2.0 * ry + rz)), dtype=f)
    kx = np.full(T.shape, f(cap * rx), dtype=f)
    ky = np.full(T.shape, f(cap * ry), dtype=f)
    q = fma32(np.full(T.shape, f(cap), dtype=f), P.astype(f), f(cap * rz * amb))
    t = T.astype(f).copy()
    for _ in range(iters):
        g = np.pad(t, 1, mode="edge")
        n, s, e, w = g[:-2, 1:-1], g[2:, 1:-1], g[1:-1, 2:], g[1:-1, :-2]
        u = fma32(kt, t, q)
        u = fma32(kx, e + w, u)
        t = fma32(ky, s + n, u)
    return t
