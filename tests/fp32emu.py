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
    """The update in fp32 in the kernel's fixed sequence (test-side check,
    independent of the CUDA code): a = fma(-2, t, s + n), b = fma(-2, t, e + w),
    d = fma(a, ry, p), d = fma(b, rx, d), d = fma(amb - t, rz, d), t' = fma(cap, d, t)."""
    k = nu.hotspot_coeffs(*T.shape) if k is None else k
    f = np.float32
    cap, rx, ry, rz, amb = f(k.cap_1), f(k.rx_1), f(k.ry_1), f(k.rz_1), f(k.amb)
    t = T.astype(np.float32).copy()
    p = P.astype(np.float32)
    m2 = np.float32(-2)
    for _ in range(iters):
        g = np.pad(t, 1, mode="edge")
        n, s, e, w = g[:-2, 1:-1], g[2:, 1:-1], g[1:-1, 2:], g[1:-1, :-2]
        ay = fma32(np.full_like(t, m2), t, s + n)
        ax = fma32(np.full_like(t, m2), t, e + w)
        d = fma32(ay, np.full_like(t, ry), p)
        d = fma32(ax, np.full_like(t, rx), d)
        d = fma32(amb - t, np.full_like(t, rz), d)
        t = fma32(np.full_like(t, cap), d, t)
    return t


