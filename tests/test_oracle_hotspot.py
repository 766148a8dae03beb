"""Pins of the HotSpot-2D oracle (oracle/hotspot.py, NEXT-3) against things
other than itself: [18]'s explicit edge/corner formulas written out as loops,
closed forms (ambient fixed point, the uniform-field geometric decay, a
linear field's zero interior Laplacian and its edge values, a single hot
cell's spread), transpose equivariance, and the paper's blocked recursion
(§IV-B) reproducing the plain sweep bit for bit."""
import numpy as np
import pytest

import nugen
from oracle import hotspot as hs

K = hs.coeffs(1024, 1024)


def grids(R, C, seed=1):
    return (nugen.fill(R, C, seed, nugen.MAT_T, "temp"), nugen.fill(R, C, seed, nugen.MAT_P, "power"))


def test_coefficients_and_stability():
    # RH2: the cell pitch is fixed, so the coefficients do not depend on the grid
    assert hs.coeffs(32768, 32768) == K
    assert K["rx_1"] == pytest.approx(0.1) and K["ry_1"] == pytest.approx(0.1)
    assert K["cap_1"] == pytest.approx(1.3653, rel=1e-4)
    assert K["rz_1"] == pytest.approx(1 / 20480, rel=1e-12)
    assert hs.stable(K)
    # [18]'s fixed 16 mm chip at 32768 cells would be unstable (why RH2 exists)
    gw = 0.016 / 32768
    cap = 0.5 * 1.75e6 * 0.0005 * gw * gw
    step = 0.001 / (3e6 / (0.5 * 0.0005 * 1.75e6))
    assert step / cap * 0.4 > 1


@pytest.mark.parametrize("R,C", [(1, 1), (1, 7), (6, 1), (2, 2), (5, 9), (16, 11)])
def test_step_matches_explicit_case_formulas(R, C):
    T, P = grids(R, C, seed=R * 31 + C)
    a = hs.step(T, P, K)
    b = hs.step_cases(T.tolist(), P.tolist(), K)
    assert np.allclose(a, b, rtol=1e-13, atol=0)


def test_ambient_fixed_point():
    T = np.full((9, 13), K["amb"])
    P = np.zeros((9, 13))
    assert np.array_equal(hs.run(T, P, 5, K), T)


def test_uniform_field_closed_form():
    T0, p, n = 330.0, 0.2, 7
    T = np.full((8, 8), T0)
    P = np.full((8, 8), p)
    c, z = K["cap_1"], K["rz_1"]
    t_star = K["amb"] + p / z
    expect = t_star + (1 - c * z) ** n * (T0 - t_star)
    assert np.allclose(hs.run(T, P, n, K), expect, rtol=1e-13)


def test_linear_field_interior_and_edges():
    R, C, a, b = 6, 10, 300.0, 0.75
    T = a + b * np.arange(C)[None, :] * np.ones((R, 1))
    P = np.zeros((R, C))
    out = hs.step(T, P, K)
    c, x, z, amb = K["cap_1"], K["rx_1"], K["rz_1"], K["amb"]
    base = T + c * (amb - T) * z
    assert np.allclose(out[:, 1:-1], base[:, 1:-1], rtol=1e-14)        # zero Laplacian
    assert np.allclose(out[:, 0], base[:, 0] + c * b * x, rtol=1e-14)   # west edge: E - T = +b
    assert np.allclose(out[:, -1], base[:, -1] - c * b * x, rtol=1e-14) # east edge: W - T = -b


def test_single_hot_cell_spread():
    R, C, d = 7, 9, 5.0
    T = np.full((R, C), K["amb"])
    T[3, 4] += d
    out = hs.step(T, np.zeros((R, C)), K) - K["amb"]
    c = K["cap_1"]
    assert out[3, 4] == pytest.approx(d * (1 - c * (2 * K["rx_1"] + 2 * K["ry_1"] + K["rz_1"])))
    assert out[2, 4] == pytest.approx(c * K["ry_1"] * d) and out[4, 4] == pytest.approx(c * K["ry_1"] * d)
    assert out[3, 3] == pytest.approx(c * K["rx_1"] * d) and out[3, 5] == pytest.approx(c * K["rx_1"] * d)
    mask = np.ones((R, C), bool)
    mask[[3, 2, 4, 3, 3], [4, 4, 4, 3, 5]] = False
    assert np.all(out[mask] == 0.0)


def test_transpose_equivariance():
    T, P = grids(12, 17, seed=3)
    a = hs.run(T, P, 3, K)
    b = hs.run(T.T, P.T, 3, K).T
    assert np.allclose(a, b, rtol=1e-13)


@pytest.mark.parametrize("R,C,iters,dim,halo", [(40, 56, 6, 16, 3), (33, 20, 5, 8, 2),
                                                (17, 17, 4, 17, 4), (50, 30, 7, 12, 7)])
def test_blocked_recursion_is_bitwise_the_plain_sweep(R, C, iters, dim, halo):
    T, P = grids(R, C, seed=R + C)
    assert np.array_equal(hs.blocked(T, P, iters, K, dim, halo), hs.run(T, P, iters, K))


def test_blocked_detects_a_too_narrow_border():
    """With borders narrower than the iterations per pass, the window's
    invalid band reaches the block: NaN shows up (the pin has teeth)."""
    T, P = grids(24, 24, seed=9)
    out = hs.blocked(T, P, 4, K, 8, 4)
    assert not np.isnan(out).any()
    # emulate a border of 1 for 2 iterations per pass by hand
    w = T[0:9 + 1, 0:9].astype(np.float64)
    bad = hs._window_step(hs._window_step(w, P[0:10, 0:9].astype(np.float64), 0, 0, 24, 24, K),
                          P[0:10, 0:9].astype(np.float64), 0, 0, 24, 24, K)
    assert np.isnan(bad[-2:, :]).any() and np.isnan(bad[:, -2:]).any()


def test_tolerance_model_against_fp32_emulation():
    """RH3: an fp32 emulation of the update (same expression, float32 at every
    step) stays within the bound after many iterations."""
    T, P = grids(32, 48, seed=4)
    k32 = {kk: np.float32(v) for kk, v in K.items()}
    t = T.astype(np.float32)
    p = P.astype(np.float32)
    for _ in range(40):     # fp32 at every operation (no fused operations in this emulation)
        g = np.pad(t, 1, mode="edge")
        n, s, e, w = g[:-2, 1:-1], g[2:, 1:-1], g[1:-1, 2:], g[1:-1, :-2]
        t = (t + k32["cap_1"] * (p + (s + n - np.float32(2) * t) * k32["ry_1"]
                                 + (e + w - np.float32(2) * t) * k32["rx_1"]
                                 + (k32["amb"] - t) * k32["rz_1"])).astype(np.float32)
    ref = hs.run(T, P, 40, K)
    err = np.abs(t.astype(np.float64) - ref).max()
    assert err <= hs.tolerance(40, np.abs(ref).max())
    assert err > 0   # fp32 really differs (the bound is exercised)


def test_expanded_form_equals_definition_and_stays_within_bound():
    """RH4 (revised): the kernel evaluates T' = kt T + kx (E + W) + ky (S + N) + q,
    q = cap_1 P + cap_1 rz_1 amb.  In fp64 that is the definition up to
    rounding; its fixed fp32 sequence (the test-side emulation of the kernel)
    stays within RH3's bound of the fp64 oracle after 256 iterations, and its
    weights are positive (a convex combination: errors do not grow)."""
    from fp32emu import emulate_fp32
    import paper_conf_ipps_chey19_b200 as nu
    T, P = grids(40, 56, seed=6)
    k = K
    kt = 1.0 - k["cap_1"] * (2 * k["rx_1"] + 2 * k["ry_1"] + k["rz_1"])
    kx, ky = k["cap_1"] * k["rx_1"], k["cap_1"] * k["ry_1"]
    assert kt > 0 and kx > 0 and ky > 0
    t = T.astype(np.float64)
    q = k["cap_1"] * P.astype(np.float64) + k["cap_1"] * k["rz_1"] * k["amb"]
    for _ in range(5):
        g = np.pad(t, 1, mode="edge")
        n, s, e, w = g[:-2, 1:-1], g[2:, 1:-1], g[1:-1, 2:], g[1:-1, :-2]
        t = kt * t + kx * (e + w) + ky * (s + n) + q
    assert np.abs(t - hs.run(T, P, 5, K)).max() <= 1e-10
    out = emulate_fp32(T, P, 256, nu.hotspot_coeffs(40, 56))
    ref = hs.run(T, P, 256, K)
    err = np.abs(out.astype(np.float64) - ref).max()
    assert 0 < err <= hs.tolerance(256, np.abs(ref).max())


def test_fma32_emulation_is_exact():
    """Pin of the test-side fma (tests/fp32emu.py) against exact rational
    arithmetic, including sums that land on float32 rounding boundaries."""
    from fractions import Fraction

    from fp32emu import fma32
    rng = np.random.default_rng(3)
    a = rng.standard_normal(3000).astype(np.float32)
    b = rng.standard_normal(3000).astype(np.float32)
    c = (rng.standard_normal(3000) * 1e-3).astype(np.float32)
    # near-midpoint cases: c = -(a*b rounded to float32) + a tiny offset
    ab32 = (a.astype(np.float64) * b.astype(np.float64)).astype(np.float32)
    c[::3] = (-ab32[::3]).astype(np.float32)
    got = fma32(a, b, c)
    for i in range(0, 3000, 5):
        exact = Fraction(float(a[i])) * Fraction(float(b[i])) + Fraction(float(c[i]))
        f = np.float32(float(exact))                 # candidate near the exact value
        cands = {float(f), float(np.nextafter(f, np.float32(np.inf))), float(np.nextafter(f, np.float32(-np.inf)))}
        dist = {v: abs(Fraction(v) - exact) for v in cands}
        m = min(dist.values())
        best = [v for v in cands if dist[v] == m]
        if len(best) > 1:                            # tie: round half to even
            best = [v for v in best if (int(np.array(v, np.float32).view(np.int32)) & 1) == 0]
        assert float(got[i]) == best[0], i
