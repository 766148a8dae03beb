"""HotSpot-2D on the B200 (NEXT-3): the sm_100a leaf and the tree runtime
(in-HBM and HOST -> HBM out-of-core, virtual siblings) against the fp64
oracle (oracle/hotspot.py) within the RH3 bound, and bit for bit against an
fp32 emulation of the update in the kernel's evaluation order; in-HBM and
out-of-core runs agree bit for bit whatever the blocks, borders and
iterations per launch."""
import ctypes

import numpy as np
import pytest
import torch

import nugen
import paper_conf_ipps_chey19_b200 as nu
from oracle import hotspot as hs
from fp32emu import emulate_fp32

pytestmark = pytest.mark.gpu
K = hs.coeffs(1024, 1024)


def grids(R, C, seed):
    return (nugen.fill(R, C, seed, nugen.MAT_T, "temp"), nugen.fill(R, C, seed, nugen.MAT_P, "power"))


def check(out, T, P, iters):
    ref = hs.run(T, P, iters, K)
    err = np.abs(out.astype(np.float64) - ref).max()
    assert err <= hs.tolerance(iters, np.abs(ref).max()), err


@pytest.mark.parametrize("R,C,iters", [(1, 1, 3), (7, 300, 8), (200, 257, 1), (333, 129, 5), (130, 70, 8)])
def test_leaf_whole_grid(R, C, iters):
    T, P = grids(R, C, seed=R * 7 + C)
    dev = torch.device("cuda", 0)
    t, p = torch.from_numpy(T).to(dev), torch.from_numpy(P).to(dev)
    o = torch.full_like(t, float("nan"))
    nu.hotspot_leaf(t, p, o, iters)
    out = o.cpu().numpy()
    check(out, T, P, iters)
    assert np.array_equal(out, emulate_fp32(T, P, iters))


@pytest.mark.parametrize("R,C,iters", [(130, 70, 8), (300, 516, 5)])
def test_leaf_caller_coefficients(R, C, iters):
    """Coefficients other than [18]'s defaults (the library specialises the
    default set into immediates; any other set is passed as kernel arguments):
    bitwise equal to the fp32 emulation with the same set, within RH3 of the
    fp64 oracle."""
    kc = nu.HotspotCoeffs(1.2, 0.11, 0.09, 1e-4, 75.0)
    kd = {n: float(getattr(kc, n)) for n in ("cap_1", "rx_1", "ry_1", "rz_1", "amb")}
    T, P = grids(R, C, seed=5 * R + C)
    dev = torch.device("cuda", 0)
    t, p = torch.from_numpy(T).to(dev), torch.from_numpy(P).to(dev)
    o = torch.full_like(t, float("nan"))
    nu.hotspot_leaf(t, p, o, iters, coeffs=kc)
    out = o.cpu().numpy()
    assert np.array_equal(out, emulate_fp32(T, P, iters, kc))
    assert not np.array_equal(out, emulate_fp32(T, P, iters))     # the set really differs
    ref = hs.run(T, P, iters, kd)
    assert np.abs(out.astype(np.float64) - ref).max() <= hs.tolerance(iters, np.abs(ref).max())


def test_leaf_sub_window_valid_region():
    """A window inside the grid: only the valid region (shrunk by `iters` on
    non-edge sides) is written, and it equals the full-grid evolution."""
    R, C, iters = 300, 400, 6
    T, P = grids(R, C, seed=11)
    full = emulate_fp32(T, P, iters)
    dev = torch.device("cuda", 0)
    for (y0, y1, x0, x1) in [(50, 200, 60, 300), (0, 120, 100, 400), (250, 300, 0, 77)]:
        t = torch.from_numpy(np.ascontiguousarray(T[y0:y1, x0:x1])).to(dev)
        p = torch.from_numpy(np.ascontiguousarray(P[y0:y1, x0:x1])).to(dev)
        o = torch.full_like(t, float("nan"))
        nu.hotspot_leaf(t, p, o, iters, gy0=y0, gx0=x0, rows=R, cols=C)
        out = o.cpu().numpy()
        vy0 = 0 if y0 == 0 else iters
        vy1 = (y1 - y0) - (0 if y1 == R else iters)
        vx0 = 0 if x0 == 0 else iters
        vx1 = (x1 - x0) - (0 if x1 == C else iters)
        assert np.array_equal(out[vy0:vy1, vx0:vx1], full[y0 + vy0:y0 + vy1, x0 + vx0:x0 + vx1])
        mask = np.ones(out.shape, bool)
        mask[vy0:vy1, vx0:vx1] = False
        assert np.isnan(out[mask]).all()            # nothing outside the valid region


def host_view(buf, rows, cols):
    return np.ctypeslib.as_array((ctypes.c_float * (rows * cols)).from_address(buf.ptr)).reshape(rows, cols)


def run_tree(R, C, iters, G=1, cap=0, coeffs=None, **opt):
    t, _ = nu.host_tree(G, cap, devices=[0] * G)
    t.finalize()
    Tb, Pb, Ob = t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0)
    T, P = host_view(Tb, R, C), host_view(Pb, R, C)
    T[...], P[...] = grids(R, C, seed=R + C)
    host_view(Ob, R, C)[...] = np.nan
    st = t.hotspot(Tb, Pb, Ob, R, C, iters, nu.hotspot_opts(**opt), coeffs=coeffs)
    out, Tc, Pc = host_view(Ob, R, C).copy(), T.copy(), P.copy()
    assert np.array_equal(T, grids(R, C, seed=R + C)[0])      # T is not modified
    t.destroy()
    return out, Tc, Pc, st


def run_in_hbm(R, C, iters, leaf_iters=0):
    T, P = grids(R, C, seed=R + C)
    dev = torch.device("cuda", 0)
    t = nu.hbm_tree(0)
    t.finalize()
    Td, Pd = torch.from_numpy(T).to(dev), torch.from_numpy(P).to(dev)
    Od = torch.full_like(Td, float("nan"))
    st = t.hotspot(t.wrap_device(0, Td.data_ptr(), Td.numel() * 4), t.wrap_device(0, Pd.data_ptr(), Pd.numel() * 4),
                   t.wrap_device(0, Od.data_ptr(), Od.numel() * 4), R, C, iters, nu.hotspot_opts(leaf_iters=leaf_iters))
    out = Od.cpu().numpy()
    t.destroy()
    return out, T, P, st


@pytest.mark.parametrize("R,C,iters,G,cap,opt", [
    (1000, 1200, 20, 1, 0, dict(block=256, halo=8)),
    (1000, 1200, 20, 2, 0, dict(block=320, halo=6, leaf_iters=3)),
    (777, 515, 13, 1, 6 << 20, dict()),
    (2048, 2048, 40, 4, 0, dict(block=512, halo=20)),
])
def test_tree_out_of_core_matches_in_hbm_and_oracle(R, C, iters, G, cap, opt):
    out, T, P, st = run_tree(R, C, iters, G, cap, **opt)
    ref_hbm, _, _, _ = run_in_hbm(R, C, iters)
    assert np.array_equal(out, ref_hbm)                  # bitwise, any blocking
    assert np.array_equal(out, emulate_fp32(T, P, iters))
    check(out, T, P, iters)
    assert st["leaf_launches"] > 0 and st["bytes_h2d"] >= 8 * R * C


def test_tree_out_of_core_caller_coefficients():
    """Caller coefficients through the tree (the plan carries them to every
    leaf launch): bitwise equal to the fp32 emulation with the same set and
    within RH3 of the fp64 oracle."""
    kc = nu.HotspotCoeffs(1.1, 0.12, 0.08, 2e-4, 70.0)
    R, C, iters = 900, 1100, 19
    out, T, P, st = run_tree(R, C, iters, 2, 0, coeffs=kc, block=256, halo=10, leaf_iters=5)
    assert np.array_equal(out, emulate_fp32(T, P, iters, kc))
    kd = {n: float(getattr(kc, n)) for n in ("cap_1", "rx_1", "ry_1", "rz_1", "amb")}
    ref = hs.run(T, P, iters, kd)
    assert np.abs(out.astype(np.float64) - ref).max() <= hs.tolerance(iters, np.abs(ref).max())


def test_in_hbm_leaf_iters_invariance():
    a = run_in_hbm(513, 640, 17, leaf_iters=8)[0]
    b = run_in_hbm(513, 640, 17, leaf_iters=1)[0]
    c = run_in_hbm(513, 640, 17, leaf_iters=5)[0]
    assert np.array_equal(a, b) and np.array_equal(a, c)


def _on_device(X, dev, layout):
    """X on the device as a row-major view: "dense" (ld = cols), "padded" (ld a
    multiple of 4 floats, base 16-B aligned: the persistent TMA kernel) or
    "offset" (base 4 bytes past an aligned one: the v5 fallback)."""
    R, C = X.shape
    if layout == "dense":
        return torch.from_numpy(np.ascontiguousarray(X)).to(dev)
    ld = (C + 3) // 4 * 4 + 4
    buf = torch.full((R + 1, ld + 1), float("nan"), device=dev)
    flat = buf.view(-1)
    off = 1 if layout == "offset" else 0
    v = flat[off:off + R * ld].view(R, ld)[:, :C]
    v.copy_(torch.from_numpy(np.ascontiguousarray(X)))
    return v


@pytest.mark.parametrize("layout", ["dense", "padded", "offset"])
@pytest.mark.parametrize("R,C,iters", [(700, 900, 8), (129, 131, 3), (1, 257, 5), (300, 2, 7), (97, 129, 8),
                                        (450, 333, 6), (1000, 1200, 8), (260, 250, 1)])
def test_leaf_bitwise_vs_emulation(R, C, iters, layout):
    """The leaf evaluates RH4's sequence per cell, so it equals the exact fp32
    emulation bit for bit — whole grids (edge tiles, tile-size boundaries at
    96 / 112 / 116 / 128 / 132 cells) and grids large enough for clamp-free interior tiles,
    through the persistent TMA kernel (aligned windows) and the v5 fallback
    (unaligned base or leading dimension)."""
    T, P = grids(R, C, seed=R + 3 * C)
    dev = torch.device("cuda", 0)
    t, p = _on_device(T, dev, layout), _on_device(P, dev, layout)
    o = _on_device(np.full((R, C), np.nan, np.float32), dev, layout)
    nu.hotspot_leaf(t, p, o, iters)
    full = emulate_fp32(T, P, iters)
    assert np.array_equal(o.cpu().numpy(), full)
    # a sub-window: only its valid region is written, equal to the full-grid evolution
    if R > 2 * iters + 2 and C > 2 * iters + 2:
        y0, y1, x0, x1 = 1, R - 1, 1, C - 1
        tw = _on_device(T[y0:y1, x0:x1], dev, layout)
        pw = _on_device(P[y0:y1, x0:x1], dev, layout)
        ow = _on_device(np.full((y1 - y0, x1 - x0), np.nan, np.float32), dev, layout)
        nu.hotspot_leaf(tw, pw, ow, iters, gy0=y0, gx0=x0, rows=R, cols=C)
        out = ow.cpu().numpy()
        assert np.array_equal(out[iters:-iters, iters:-iters], full[y0 + iters:y1 - iters, x0 + iters:x1 - iters])


def test_leaf_concurrent_streams_and_tile_counts():
    """The persistent leaf claims tiles from a per-(device, stream) counter that
    its last CTA re-arms: launches on several streams at once, back-to-back
    launches on one stream, and windows whose tile-column count equals half the
    grid of CTAs (the shape that once concentrated a clamped edge column on two
    CTAs) all give the emulation's result bit for bit."""
    dev = torch.device("cuda", 0)
    n_sm = torch.cuda.get_device_properties(dev).multi_processor_count
    iters = 8
    # tile columns = ceil((wn - iters) / 112) for a window at the grid's west edge
    shapes = [(300, 112 * (n_sm // 2) + iters - 4), (260, 112 * (n_sm // 2) + 20), (390, 1000), (129, 517)]
    cases = []
    for i, (R, C) in enumerate(shapes):
        T, P = grids(R, C, seed=40 + i)
        t, p = torch.from_numpy(T).to(dev), torch.from_numpy(P).to(dev)
        cases.append((T, P, t, p, [torch.full_like(t, float("nan")) for _ in range(2)]))
    streams = [torch.cuda.Stream(dev) for _ in cases]
    torch.cuda.synchronize(dev)
    for rep in range(3):                       # counters must be re-armed after every launch
        for (T, P, t, p, outs), s in zip(cases, streams):
            with torch.cuda.stream(s):
                nu.hotspot_leaf(t, p, outs[0], iters, stream=s)
                nu.hotspot_leaf(outs[0], p, outs[1], iters, stream=s)
    torch.cuda.synchronize(dev)
    for T, P, t, p, outs in cases:
        assert np.array_equal(outs[1].cpu().numpy(), emulate_fp32(T, P, 2 * iters))
