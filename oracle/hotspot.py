"""ORACLE — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

HotSpot-2D thermal simulation, the paper's stencil case study (§IV-B,
P:307-325; S§8(f) NEXT-3), as plain fp64 numpy.  Shares no code with the CUDA
path and never imports it.

The paper names the benchmark (HotSpot-2D [18]) but does not
print its update; the update below is [18]'s explicit scheme restated
(reading RH1), with every grid cell (r, c):

    T'[r,c] = T[r,c] + cap_1 * ( P[r,c]
                                 + (T[S] + T[N] - 2 T[r,c]) * ry_1
                                 + (T[E] + T[W] - 2 T[r,c]) * rx_1
                                 + (amb - T[r,c]) * rz_1 )

N/S = rows r-1 / r+1, W/E = columns c-1 / c+1; a neighbour outside the grid
is the cell itself (the edge and corner cases of [18] are exactly this clamp;
`step_cases` writes them out one by one as an independent pin).

Coefficients (RH1, [18]'s chip model):  Cap = 0.5 * 1.75e6 * t_chip * gw * gh,
Rx = gw / (2 * 100 * t_chip * gh), Ry = gh / (2 * 100 * t_chip * gw),
Rz = t_chip / (100 * gh * gw), max_slope = 3e6 / (0.5 * t_chip * 1.75e6),
step = 0.001 / max_slope, t_chip = 0.0005 m, amb = 80; cap_1 = step / Cap,
rx_1 = 1 / Rx, ry_1 = 1 / Ry, rz_1 = 1 / Rz.  [18] fixes a 16 mm chip, so the
cell pitch shrinks with the grid and the explicit scheme becomes unstable
above ~1448 cells per side (cap_1 * (2 rx_1 + 2 ry_1) > 1).  Reading RH2: the
cell pitch is fixed at [18]'s 1024-cell value (gw = gh = 16 mm / 1024), so
the coefficients are the same for every grid and the scheme is stable at the
paper's 16k and 32k grids.

  * `coeffs`      — the five coefficients in fp64 (RH1, RH2);
  * `step`/`run`  — the definition, vectorised with an edge clamp (O1 analog);
  * `step_cases`  — [18]'s nine cases (4 corners, 4 edges, interior) as plain
                    Python loops: an independent formulation for small grids;
  * `blocked`     — §IV-B's recursive step literally: sub-blocks of
                    dim x dim with their borders moved down a level, `halo`
                    iterations there, the block copied back up (O2 analog);
  * `tolerance`   — the fp32 acceptance bound (RH3).
"""
from __future__ import annotations

import numpy as np

T_CHIP = 0.0005
K_SI = 100.0
SPEC_HEAT_SI = 1.75e6
FACTOR_CHIP = 0.5
MAX_PD = 3.0e6
PRECISION = 0.001
AMB_TEMP = 80.0
PITCH = 0.016 / 1024          # RH2: [18]'s cell pitch at 1024 cells per side


def coeffs(rows: int, cols: int) -> dict:
    """The update's coefficients in fp64 (RH1 with the RH2 cell pitch).
    rows/cols only enter through the pitch, which RH2 fixes."""
    gh = PITCH
    gw = PITCH
    cap = FACTOR_CHIP * SPEC_HEAT_SI * T_CHIP * gw * gh
    rx = gw / (2.0 * K_SI * T_CHIP * gh)
    ry = gh / (2.0 * K_SI * T_CHIP * gw)
    rz = T_CHIP / (K_SI * gh * gw)
    max_slope = MAX_PD / (FACTOR_CHIP * T_CHIP * SPEC_HEAT_SI)
    step = PRECISION / max_slope
    return {"cap_1": step / cap, "rx_1": 1.0 / rx, "ry_1": 1.0 / ry, "rz_1": 1.0 / rz,
            "amb": AMB_TEMP}


def _update(t, p, n, s, e, w, k):
    return t + k["cap_1"] * (p + (s + n - 2.0 * t) * k["ry_1"] + (e + w - 2.0 * t) * k["rx_1"]
                             + (k["amb"] - t) * k["rz_1"])


def step(T, P, k) -> np.ndarray:
    """One iteration over the whole grid, fp64, neighbours clamped at the edges."""
    t = np.asarray(T, dtype=np.float64)
    p = np.asarray(P, dtype=np.float64)
    g = np.pad(t, 1, mode="edge")
    return _update(t, p, g[:-2, 1:-1], g[2:, 1:-1], g[1:-1, 2:], g[1:-1, :-2], k)


def run(T, P, iters: int, k) -> np.ndarray:
    t = np.asarray(T, dtype=np.float64)
    for _ in range(iters):
        t = step(t, P, k)
    return t


def step_cases(T, P, k) -> np.ndarray:
    """[18]'s explicit per-case formulas (corners, edges, interior), loops.
    A missing neighbour drops its (X - T) term instead of being clamped."""
    R, C = len(T), len(T[0])
    out = np.empty((R, C), dtype=np.float64)
    cap_1, rx_1, ry_1, rz_1, amb = k["cap_1"], k["rx_1"], k["ry_1"], k["rz_1"], k["amb"]
    for r in range(R):
        for c in range(C):
            t = float(T[r][c])
            d = float(P[r][c]) + (amb - t) * rz_1
            if r > 0:
                d += (float(T[r - 1][c]) - t) * ry_1
            if r < R - 1:
                d += (float(T[r + 1][c]) - t) * ry_1
            if c > 0:
                d += (float(T[r][c - 1]) - t) * rx_1
            if c < C - 1:
                d += (float(T[r][c + 1]) - t) * rx_1
            out[r, c] = t + cap_1 * d
    return out


def _window_step(t, p, gy0, gx0, R, C, k):
    """One iteration on a window at global (gy0, gx0) of an R x C grid: global
    edges clamp, window edges inside the grid have unknown outer neighbours
    (NaN), so the valid region shrinks by one per iteration on those sides."""
    m, n = t.shape
    g = np.full((m + 2, n + 2), np.nan)
    g[1:-1, 1:-1] = t
    if gy0 == 0:
        g[0, 1:-1] = t[0]
    if gy0 + m == R:
        g[-1, 1:-1] = t[-1]
    if gx0 == 0:
        g[1:-1, 0] = t[:, 0]
    if gx0 + n == C:
        g[1:-1, -1] = t[:, -1]
    return _update(t, p, g[:-2, 1:-1], g[2:, 1:-1], g[1:-1, 2:], g[1:-1, :-2], k)


def blocked(T, P, iters: int, k, dim: int, halo: int) -> np.ndarray:
    """§IV-B literally: per pass of `halo` iterations, divide the
    grid into dim x dim sub-blocks; for each, copy the block with its four
    borders (halo wide, clipped at the grid edge) and the matching power down
    a level, iterate there, and copy the block's result back up."""
    cur = np.asarray(T, dtype=np.float64).copy()
    Pd = np.asarray(P, dtype=np.float64)
    R, C = cur.shape
    done = 0
    while done < iters:
        h = min(halo, iters - done)
        nxt = np.empty_like(cur)
        for y0 in range(0, R, dim):
            for x0 in range(0, C, dim):
                y1, x1 = min(R, y0 + dim), min(C, x0 + dim)
                wy0, wx0 = max(0, y0 - h), max(0, x0 - h)
                wy1, wx1 = min(R, y1 + h), min(C, x1 + h)
                tw = cur[wy0:wy1, wx0:wx1].copy()          # data_down: block + borders
                pw = Pd[wy0:wy1, wx0:wx1].copy()
                for _ in range(h):
                    tw = _window_step(tw, pw, wy0, wx0, R, C, k)
                nxt[y0:y1, x0:x1] = tw[y0 - wy0:y1 - wy0, x0 - wx0:x1 - wx0]   # data_up
        cur = nxt
        done += h
    return cur


def tolerance(iters: int, tmax: float) -> float:
    """RH3: fp32 bound for |T_gpu - T_ref| after `iters` iterations.  The
    update is a convex combination (weights >= 0, checked by
    `stable`) plus a source term, so per-iteration rounding errors do not grow;
    each iteration adds < 4 ulp-sized errors (T + delta rounding, cancellation
    in the neighbour sums) of at most 2^-23 max|T|."""
    return 4.0 * max(1, iters) * 2.0 ** -23 * tmax


def stable(k) -> bool:
    """Explicit-scheme weights are nonnegative: 1 - cap_1 (2 rx_1 + 2 ry_1 + rz_1) >= 0."""
    return 1.0 - k["cap_1"] * (2 * k["rx_1"] + 2 * k["ry_1"] + k["rz_1"]) >= 0.0
