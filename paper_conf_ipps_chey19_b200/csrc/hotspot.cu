// HotSpot-2D leaf (S§8(f) NEXT-3; §IV-B): the explicit
// thermal update of [18] (reading RH1, coefficients RH2) on a window
// of the grid resident in HBM, several iterations per launch.
//
// The paper's leaf loads a block and its borders into (block+2)^2 local-memory
// arrays and does one iteration.  Here a CTA loads its 64 x 64 output
// tile plus an `iters`-wide border of temperature and power into shared
// memory once and performs all `iters` iterations there (the valid region
// shrinks by one cell per iteration on every side that is not a grid edge),
// so HBM is read once and written once per `iters` iterations.
//
// Arithmetic contract (RH4): every cell update is the fixed fp32
// sequence (round-to-nearest, fma = one rounding)
//     a = fma(-2, t, s + n);  b = fma(-2, t, e + w)
//     d = fma(a, ry_1, p);  d = fma(b, rx_1, d);  d = fma(amb - t, rz_1, d)
//     t' = fma(cap_1, d, t)
// written with __fadd_rn/__fmaf_rn so the compiler cannot reassociate or
// re-fuse it: 3 FADD + 6 FFMA per update.  The result of a cell is therefore
// independent of tiling, iterations per launch and launch order: in-HBM and
// out-of-core runs agree bit for bit, and so does an exact fp32 emulation.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "northup_internal.h"

namespace nu {
namespace hs {

constexpr int kTY = 64, kTX = 64;   // output tile per CTA
constexpr int kWX = 32, kWY = 16;   // 512 threads as 32 x 16
constexpr int kThreads = kWX * kWY;

struct Args {
  const float* tin;
  const float* pw;
  float* tout;
  int64_t ldt, ldp, ldo;
  int64_t wm, wn;            // window rows / cols
  int64_t gy0, gx0;          // window origin in the grid
  int64_t R, C;              // grid
  int64_t vy0, vy1, vx0, vx1;  // valid output region (window coordinates)
  int iters;
  float cap_1, rx_1, ry_1, rz_1, amb;
};

__device__ __forceinline__ float update(float t, float p, float n, float s, float e, float w,
                                        const Args& a) {
  const float ay = __fmaf_rn(-2.0f, t, __fadd_rn(s, n));
  const float ax = __fmaf_rn(-2.0f, t, __fadd_rn(e, w));
  float d = __fmaf_rn(ay, a.ry_1, p);
  d = __fmaf_rn(ax, a.rx_1, d);
  d = __fmaf_rn(__fsub_rn(a.amb, t), a.rz_1, d);
  return __fmaf_rn(a.cap_1, d, t);
}

// 4-byte asynchronous global -> shared copies (LDGSTS): every element of the
// tile is in flight at once instead of one load per thread per loop trip.
__device__ __forceinline__ void cp_async4(float* smem, const float* gmem) {
  const unsigned sa = static_cast<unsigned>(__cvta_generic_to_shared(smem));
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
}

__global__ void __launch_bounds__(kThreads) hotspot_kernel(Args a) {
  extern __shared__ float sm[];
  const int it = a.iters;
  const int SX = kTX + 2 * it, SY = kTY + 2 * it;
  float* cur = sm;
  float* nxt = sm + SY * SX;
  float* pwr = sm + 2 * SY * SX;
  const int tx = threadIdx.x, ty = threadIdx.y;

  const int64_t ty0 = a.vy0 + static_cast<int64_t>(blockIdx.y) * kTY;
  const int64_t tx0 = a.vx0 + static_cast<int64_t>(blockIdx.x) * kTX;
  const int64_t ty1 = min(ty0 + kTY, a.vy1), tx1 = min(tx0 + kTX, a.vx1);
  const int64_t sy0 = max(ty0 - it, int64_t(0)), sy1 = min(ty1 + it, a.wm);
  const int64_t sx0 = max(tx0 - it, int64_t(0)), sx1 = min(tx1 + it, a.wn);
  const int hy = static_cast<int>(sy1 - sy0), hx = static_cast<int>(sx1 - sx0);

  // data_down HBM -> SMEM: the tile with its borders (coalesced rows, async)
  for (int y = ty; y < hy; y += kWY) {
    const float* trow = a.tin + (sy0 + y) * a.ldt + sx0;
    const float* prow = a.pw + (sy0 + y) * a.ldp + sx0;
    for (int x = tx; x < hx; x += kWX) {
      cp_async4(&cur[y * SX + x], trow + x);
      cp_async4(&pwr[y * SX + x], prow + x);
    }
  }
  cp_async_wait_all();
  __syncthreads();

  // sides of the shared-memory region that are grid edges (clamped, never shrink)
  const bool top = a.gy0 + sy0 == 0, bot = a.gy0 + sy1 == a.R;
  const bool lef = a.gx0 + sx0 == 0, rig = a.gx0 + sx1 == a.C;
  for (int k = 1; k <= it; ++k) {
    const int y0 = top ? 0 : k, y1 = bot ? hy : hy - k;
    const int x0 = lef ? 0 : k, x1 = rig ? hx : hx - k;
    for (int y = y0 + ty; y < y1; y += kWY) {
      const int yn = y > 0 ? y - 1 : 0;            // y == 0 only when `top` (clamp)
      const int ys = y < hy - 1 ? y + 1 : y;       // y == hy - 1 only when `bot`
      for (int x = x0 + tx; x < x1; x += kWX) {
        const int xw = x > 0 ? x - 1 : 0;
        const int xe = x < hx - 1 ? x + 1 : x;
        nxt[y * SX + x] = update(cur[y * SX + x], pwr[y * SX + x], cur[yn * SX + x], cur[ys * SX + x],
                                 cur[y * SX + xe], cur[y * SX + xw], a);
      }
    }
    __syncthreads();
    float* t = cur;
    cur = nxt;
    nxt = t;
  }

  // data_up SMEM -> HBM: the tile
  const int oy = static_cast<int>(ty0 - sy0), ox = static_cast<int>(tx0 - sx0);
  const int ny = static_cast<int>(ty1 - ty0), nx = static_cast<int>(tx1 - tx0);
  for (int y = ty; y < ny; y += kWY) {
    float* orow = a.tout + (ty0 + y) * a.ldo + tx0;
    for (int x = tx; x < nx; x += kWX) orow[x] = cur[(oy + y) * SX + ox + x];
  }
}

// ---------------------------------------------------------------------------
// v2: register-blocked.  A CTA owns a region of RH = NWY*RPT rows x RW = NWX*32
// columns; thread (lane, warp) keeps RPT consecutive cells of one column (and
// their power) in registers for all iterations.  Per iteration:
//   * N/S inside the segment come from registers; across segments each thread
//     publishes its top and bottom cell in shared memory;
//   * E/W come from warp shuffles; lanes 0 / 31 take the neighbouring warp's
//     edge column from shared memory;
//   * one __syncthreads (the exchange arrays are double-buffered by parity).
// Grid-edge neighbours are clamped per cell, exactly as in v1, and the update
// is the same function, so v2 is bitwise equal to v1 (tested).
template <int RPT, int NWX, int NWY>
__global__ void __launch_bounds__(NWX * NWY * 32, 1) hotspot_kernel_v2(Args a) {
  constexpr int RW = NWX * 32, RH = NWY * RPT;
  __shared__ float tops[2][NWY][RW], bots[2][NWY][RW];
  __shared__ float colL[2][NWX][RH], colR[2][NWX][RH];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int sx = warp % NWX, gyi = warp / NWX;
  const int h = a.iters;
  const int OTY = RH - 2 * h, OTX = RW - 2 * h;
  const int64_t oy0 = a.vy0 + static_cast<int64_t>(blockIdx.y) * OTY;
  const int64_t ox0 = a.vx0 + static_cast<int64_t>(blockIdx.x) * OTX;
  const int64_t ry = oy0 - h, rx = ox0 - h;        // region origin (window coordinates)
  const int x = sx * 32 + lane;                    // column inside the region
  const int64_t wx = rx + x;                       // window column
  const int64_t gcol = a.gx0 + wx;                 // grid column
  const int r0 = gyi * RPT;                        // first row of this segment
  const bool xin = wx >= 0 && wx < a.wn;

  float v[RPT], p[RPT];
#pragma unroll
  for (int r = 0; r < RPT; ++r) {
    const int64_t wy = ry + r0 + r;
    const bool in = xin && wy >= 0 && wy < a.wm;
    v[r] = in ? __ldg(a.tin + wy * a.ldt + wx) : 0.0f;
    p[r] = in ? __ldg(a.pw + wy * a.ldp + wx) : 0.0f;
  }
  // segment rows r with grid row 0 / R - 1 (clamped neighbours); else out of range
  const int rtop = static_cast<int>(-(a.gy0 + ry + r0));
  const int rbot = static_cast<int>(a.R - 1 - (a.gy0 + ry + r0));
  const bool wclamp = gcol == 0, eclamp = gcol == a.C - 1;

  for (int k = 0; k < h; ++k) {
    const int b = k & 1;
    tops[b][gyi][x] = v[0];
    bots[b][gyi][x] = v[RPT - 1];
    if (lane == 0) {
#pragma unroll
      for (int r = 0; r < RPT; ++r) colL[b][sx][r0 + r] = v[r];
    }
    if (lane == 31) {
#pragma unroll
      for (int r = 0; r < RPT; ++r) colR[b][sx][r0 + r] = v[r];
    }
    __syncthreads();
    const float n0 = gyi > 0 ? bots[b][gyi - 1][x] : v[0];
    const float sL = gyi < NWY - 1 ? tops[b][gyi + 1][x] : v[RPT - 1];
    // in place, top to bottom: `above` keeps the old value of the row above
    float above = n0;
#pragma unroll
    for (int r = 0; r < RPT; ++r) {
      const float c = v[r];
      float w = __shfl_up_sync(0xffffffffu, c, 1);
      float e = __shfl_down_sync(0xffffffffu, c, 1);
      if (lane == 0) w = sx > 0 ? colR[b][sx - 1][r0 + r] : c;
      if (lane == 31) e = sx < NWX - 1 ? colL[b][sx + 1][r0 + r] : c;
      float n = above;
      float s = r < RPT - 1 ? v[r + 1] : sL;
      if (r == rtop) n = c;                        // grid-edge clamps (as v1)
      if (r == rbot) s = c;
      if (wclamp) w = c;
      if (eclamp) e = c;
      v[r] = update(c, p[r], n, s, e, w, a);
      above = c;
    }
  }

  // the output tile: rows [oy0, oy0 + OTY) x cols [ox0, ox0 + OTX) within the valid region
  if (wx < ox0 || wx >= min(ox0 + OTX, a.vx1)) return;
  const int64_t ylo = oy0, yhi = min(oy0 + OTY, a.vy1);
#pragma unroll
  for (int r = 0; r < RPT; ++r) {
    const int64_t wy = ry + r0 + r;
    if (wy >= ylo && wy < yhi) a.tout[wy * a.ldo + wx] = v[r];
  }
}

// ---------------------------------------------------------------------------
// v3: register runs + shared-memory plane.  A CTA owns a region of
// RH = NWY*V rows x RW = NWX*32 columns (plus a one-cell apron in shared
// memory).  Thread (lane, warp) keeps V consecutive cells of column
// x = 32*(warp % NWX) + lane, and their power, in registers for all the
// launch's iterations.  Per iteration it reads the W/E neighbours of its V
// cells and the cells above / below its run from the current plane, computes
// V updates, writes them to the next plane, and the CTA synchronises once
// (two planes alternate).  CTAs whose region touches no grid edge run the
// clamp-free body; edge CTAs clamp per cell exactly as v1, so v3 is bitwise
// equal to v1 (tested).
template <int V, int NWX, int NWY, bool EDGE>
__device__ __forceinline__ void v3_iterate(const Args& a, float* __restrict__ pl0, float* __restrict__ pl1,
                                           float (&v)[V], const float (&p)[V], int x, int r0, int rtop,
                                           int rbot, bool wclamp, bool eclamp) {
  constexpr int SW = NWX * 32 + 2;   // plane row stride (apron columns 0 and SW - 1)
  float* cur = pl0;
  float* nxt = pl1;
  for (int k = 0; k < a.iters; ++k) {
    const float* crow = cur + (r0 + 1) * SW + (x + 1);   // this thread's first cell
    float above = crow[-SW];
    const float below = crow[V * SW];
#pragma unroll
    for (int r = 0; r < V; ++r) {
      const float c = v[r];
      float n = above;
      float s = r < V - 1 ? v[r + 1] : below;
      float w = crow[r * SW - 1];
      float e = crow[r * SW + 1];
      if (EDGE) {
        if (r == rtop) n = c;
        if (r == rbot) s = c;
        if (wclamp) w = c;
        if (eclamp) e = c;
      }
      v[r] = update(c, p[r], n, s, e, w, a);
      nxt[(r0 + 1 + r) * SW + x + 1] = v[r];
      above = c;
    }
    __syncthreads();
    float* t = cur;
    cur = nxt;
    nxt = t;
  }
}

#ifndef NU_HS_V3_MINB
#define NU_HS_V3_MINB 1
#endif
template <int V, int NWX, int NWY>
__global__ void __launch_bounds__(NWX * NWY * 32, NU_HS_V3_MINB) hotspot_kernel_v3(Args a) {
  constexpr int RW = NWX * 32, RH = NWY * V, SW = RW + 2, SH = RH + 2;
  extern __shared__ float sm3[];
  float* pl0 = sm3;
  float* pl1 = sm3 + SH * SW;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int x = (warp % NWX) * 32 + lane, r0 = (warp / NWX) * V;
  const int h = a.iters;
  const int OTY = RH - 2 * h, OTX = RW - 2 * h;
  const int64_t oy0 = a.vy0 + static_cast<int64_t>(blockIdx.y) * OTY;
  const int64_t ox0 = a.vx0 + static_cast<int64_t>(blockIdx.x) * OTX;
  const int64_t ry = oy0 - h, rx = ox0 - h;        // region origin (window coordinates)
  const int64_t wx = rx + x;
  const bool xin = wx >= 0 && wx < a.wn;
  float v[V], p[V];
#pragma unroll
  for (int r = 0; r < V; ++r) {
    const int64_t wy = ry + r0 + r;
    const bool in = xin && wy >= 0 && wy < a.wm;
    v[r] = in ? __ldg(a.tin + wy * a.ldt + wx) : 0.0f;
    p[r] = in ? __ldg(a.pw + wy * a.ldp + wx) : 0.0f;
  }
#pragma unroll
  for (int r = 0; r < V; ++r) pl0[(r0 + 1 + r) * SW + x + 1] = v[r];
  __syncthreads();
  // does the region touch a grid edge?  (uniform per CTA)
  const int64_t gy_top = a.gy0 + ry, gx_left = a.gx0 + rx;
  const bool edge = gy_top <= 0 || gy_top + RH >= a.R || gx_left <= 0 || gx_left + RW >= a.C;
  if (edge) {
    const int rtop = static_cast<int>(-(gy_top + r0));
    const int rbot = static_cast<int>(a.R - 1 - (gy_top + r0));
    const int64_t gcol = gx_left + x;
    v3_iterate<V, NWX, NWY, true>(a, pl0, pl1, v, p, x, r0, rtop, rbot, gcol == 0, gcol == a.C - 1);
  } else {
    v3_iterate<V, NWX, NWY, false>(a, pl0, pl1, v, p, x, r0, 0, 0, false, false);
  }
  // store: recompute the coordinates (keeps them out of the iteration's registers)
  const int64_t oy = a.vy0 + static_cast<int64_t>(blockIdx.y) * OTY;
  const int64_t ox = a.vx0 + static_cast<int64_t>(blockIdx.x) * OTX;
  const int64_t sx = ox - h + x;
  if (sx < ox || sx >= min(ox + OTX, a.vx1)) return;
  const int ylo = h - r0, yhi = static_cast<int>(min(oy + OTY, a.vy1) - (oy - h)) - r0;
  float* out = a.tout + (oy - h + r0) * a.ldo + sx;
#pragma unroll
  for (int r = 0; r < V; ++r)
    if (r >= ylo && r < yhi) out[r * a.ldo] = v[r];
}

// ---------------------------------------------------------------------------
// v4: v3 with packed fp32x2 arithmetic (sm_100 FADD2 / FFMA2).  Thread
// (lane, warp) keeps the same V-cell column run as v3, held as V/2 pairs
// (row j, row j + V/2) in 64-bit registers, so one packed instruction updates
// two cells.  The shared-memory planes store the runs in the same pair layout
// (pair-row j of run `seg` at pair-row seg*V/2 + j + 1), so the W/E neighbour
// pairs are aligned 8-byte loads and the new pair one 8-byte store.  Each lane
// of FADD2/FFMA2 is an IEEE round-to-nearest add / fused multiply-add, and
// amb - t is formed as fma(-1, t, amb) (one rounding of the exact difference),
// so every cell follows the RH4 sequence bit for bit: v4 equals v1-v3.
__device__ __forceinline__ float2 update2(float2 t, float2 p, float2 n, float2 s, float2 e, float2 w,
                                          float2 ry, float2 rx, float2 rz, float2 cap, float2 amb) {
  const float2 m2 = make_float2(-2.0f, -2.0f), m1 = make_float2(-1.0f, -1.0f);
  const float2 ay = __ffma2_rn(m2, t, __fadd2_rn(s, n));
  const float2 ax = __ffma2_rn(m2, t, __fadd2_rn(e, w));
  float2 d = __ffma2_rn(ay, ry, p);
  d = __ffma2_rn(ax, rx, d);
  d = __ffma2_rn(__ffma2_rn(m1, t, amb), rz, d);
  return __ffma2_rn(cap, d, t);
}

template <int V, int NWX, int NWY, bool EDGE>
__device__ __forceinline__ void v4_iterate(const Args& a, float2* __restrict__ pl0, float2* __restrict__ pl1,
                                           float2 (&v)[V / 2], const float2 (&p)[V / 2], int x, int pr0,
                                           int rtop, int rbot, bool wclamp, bool eclamp) {
  constexpr int SW = NWX * 32 + 2, H = V / 2;
  const float2 ry = make_float2(a.ry_1, a.ry_1), rx = make_float2(a.rx_1, a.rx_1);
  const float2 rz = make_float2(a.rz_1, a.rz_1), cap = make_float2(a.cap_1, a.cap_1);
  const float2 amb = make_float2(a.amb, a.amb);
  float2* cur = pl0;
  float2* nxt = pl1;
  for (int k = 0; k < a.iters; ++k) {
    const float2* crow = cur + pr0 * SW + (x + 1);   // this thread's first pair
    const float above = crow[-SW].y;                 // row -1 of the run
    const float below = crow[H * SW].x;              // row V of the run
    float2 prev = make_float2(above, v[H - 1].x);    // north pair of pair 0
    const float mid = v[0].y;                        // row H (south of row H - 1), pre-update
#pragma unroll
    for (int j = 0; j < H; ++j) {
      const float2 c = v[j];
      float2 n = prev;
      float2 s = j < H - 1 ? v[j + 1] : make_float2(mid, below);
      float2 w = crow[j * SW - 1];
      float2 e = crow[j * SW + 1];
      if (EDGE) {
        if (j == rtop) n.x = c.x;
        if (j + H == rtop) n.y = c.y;
        if (j == rbot) s.x = c.x;
        if (j + H == rbot) s.y = c.y;
        if (wclamp) w = c;
        if (eclamp) e = c;
      }
      v[j] = update2(c, p[j], n, s, e, w, ry, rx, rz, cap, amb);
      nxt[(pr0 + j) * SW + x + 1] = v[j];
      prev = c;
    }
    __syncthreads();
    float2* t = cur;
    cur = nxt;
    nxt = t;
  }
}

#ifndef NU_HS_V4_MINB
#define NU_HS_V4_MINB 1
#endif
template <int V, int NWX, int NWY>
__global__ void __launch_bounds__(NWX * NWY * 32, NU_HS_V4_MINB) hotspot_kernel_v4(Args a) {
  constexpr int RW = NWX * 32, RH = NWY * V, H = V / 2, SW = RW + 2, SPR = NWY * H + 2;
  extern __shared__ float2 sm4[];
  float2* pl0 = sm4;
  float2* pl1 = sm4 + SPR * SW;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int seg = warp / NWX;
  const int x = (warp % NWX) * 32 + lane, r0 = seg * V, pr0 = seg * H + 1;
  const int h = a.iters;
  const int OTY = RH - 2 * h, OTX = RW - 2 * h;
  const int64_t oy0 = a.vy0 + static_cast<int64_t>(blockIdx.y) * OTY;
  const int64_t ox0 = a.vx0 + static_cast<int64_t>(blockIdx.x) * OTX;
  const int64_t ry = oy0 - h, rx = ox0 - h;        // region origin (window coordinates)
  const int64_t wx = rx + x;
  const bool xin = wx >= 0 && wx < a.wn;
  float2 v[H], p[H];
#pragma unroll
  for (int j = 0; j < H; ++j) {
    const int64_t wy0 = ry + r0 + j, wy1 = wy0 + H;
    const bool in0 = xin && wy0 >= 0 && wy0 < a.wm, in1 = xin && wy1 >= 0 && wy1 < a.wm;
    v[j] = make_float2(in0 ? __ldg(a.tin + wy0 * a.ldt + wx) : 0.0f, in1 ? __ldg(a.tin + wy1 * a.ldt + wx) : 0.0f);
    p[j] = make_float2(in0 ? __ldg(a.pw + wy0 * a.ldp + wx) : 0.0f, in1 ? __ldg(a.pw + wy1 * a.ldp + wx) : 0.0f);
  }
#pragma unroll
  for (int j = 0; j < H; ++j) pl0[(pr0 + j) * SW + x + 1] = v[j];
  __syncthreads();
  const int64_t gy_top = a.gy0 + ry, gx_left = a.gx0 + rx;
  const bool edge = gy_top <= 0 || gy_top + RH >= a.R || gx_left <= 0 || gx_left + RW >= a.C;
  if (edge) {
    const int rtop = static_cast<int>(-(gy_top + r0));
    const int rbot = static_cast<int>(a.R - 1 - (gy_top + r0));
    const int64_t gcol = gx_left + x;
    v4_iterate<V, NWX, NWY, true>(a, pl0, pl1, v, p, x, pr0, rtop, rbot, gcol == 0, gcol == a.C - 1);
  } else {
    v4_iterate<V, NWX, NWY, false>(a, pl0, pl1, v, p, x, pr0, 0, 0, false, false);
  }
  const int64_t oy = a.vy0 + static_cast<int64_t>(blockIdx.y) * OTY;
  const int64_t ox = a.vx0 + static_cast<int64_t>(blockIdx.x) * OTX;
  const int64_t sx = ox - h + x;
  if (sx < ox || sx >= min(ox + OTX, a.vx1)) return;
  const int ylo = h - r0, yhi = static_cast<int>(min(oy + OTY, a.vy1) - (oy - h)) - r0;
  float* out = a.tout + (oy - h + r0) * a.ldo + sx;
#pragma unroll
  for (int j = 0; j < H; ++j) {
    if (j >= ylo && j < yhi) out[j * a.ldo] = v[j].x;
    if (j + H >= ylo && j + H < yhi) out[(j + H) * a.ldo] = v[j].y;
  }
}

#ifndef NU_HS_V3_V
#define NU_HS_V3_V 16
#endif
#ifndef NU_HS_V3_NWY
#define NU_HS_V3_NWY 8
#endif
constexpr int kV3V = NU_HS_V3_V, kV3NWX = 4, kV3NWY = NU_HS_V3_NWY;
#ifndef NU_HS_V4_NWX
#define NU_HS_V4_NWX 4
#endif
#ifndef NU_HS_V4_NWY
#define NU_HS_V4_NWY 8
#endif
#ifndef NU_HS_V4_V
#define NU_HS_V4_V 16
#endif
constexpr int kV4V = NU_HS_V4_V, kV4NWX = NU_HS_V4_NWX, kV4NWY = NU_HS_V4_NWY;

#ifndef NU_HS_RPT
#define NU_HS_RPT 32
#endif
#ifndef NU_HS_NWY
#define NU_HS_NWY 3
#endif
constexpr int kRPT = NU_HS_RPT, kNWX = 4, kNWY = NU_HS_NWY;   // 96 x 128 region, 384 threads

}  // namespace hs

int hotspot_max_iters_per_launch() { return kHotspotMaxIters; }

void hotspot_preload() {
  using namespace hs;
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, hotspot_kernel);
  cudaFuncGetAttributes(&fa, hotspot_kernel_v2<kRPT, kNWX, kNWY>);
  cudaFuncGetAttributes(&fa, hotspot_kernel_v3<kV3V, kV3NWX, kV3NWY>);
  cudaFuncGetAttributes(&fa, hotspot_kernel_v4<kV4V, kV4NWX, kV4NWY>);
}

static int hotspot_variant() {
  // read per launch (a getenv next to a kernel launch), so tests can switch leaves
  const char* e = getenv("NORTHUP_HS_LEAF");
  return (e && e[0] >= '1' && e[0] <= '4') ? e[0] - '0' : 3;   // 1, 2, 3: earlier leaves (DESIGN)
}

int hotspot_launch(const float* tin, int64_t ldt, const float* pw, int64_t ldp, float* tout,
                   int64_t ldo, int64_t wm, int64_t wn, int64_t gy0, int64_t gx0, int64_t R,
                   int64_t C, int iters, const float coef[5], cudaStream_t stream) {
  using namespace hs;
  if (wm < 0 || wn < 0 || R < 0 || C < 0 || gy0 < 0 || gx0 < 0 || gy0 + wm > R || gx0 + wn > C)
    return fail(NU_EINVAL, "hotspot window [%lld,%lld)x[%lld,%lld) outside the %lldx%lld grid",
                (long long)gy0, (long long)(gy0 + wm), (long long)gx0, (long long)(gx0 + wn),
                (long long)R, (long long)C);
  if (iters < 1 || iters > kHotspotMaxIters)
    return fail(NU_EINVAL, "hotspot iterations per launch must be in [1, %d]", kHotspotMaxIters);
  if (wm == 0 || wn == 0) return 0;
  if (!tin || !pw || !tout) return fail(NU_EINVAL, "NULL hotspot operand");
  if (ldt < wn || ldp < wn || ldo < wn) return fail(NU_EINVAL, "hotspot leading dimension below width");
  Args a{};
  a.tin = tin;
  a.pw = pw;
  a.tout = tout;
  a.ldt = ldt;
  a.ldp = ldp;
  a.ldo = ldo;
  a.wm = wm;
  a.wn = wn;
  a.gy0 = gy0;
  a.gx0 = gx0;
  a.R = R;
  a.C = C;
  a.iters = iters;
  // valid output region: `iters` in from every window side that is not a grid edge
  a.vy0 = gy0 == 0 ? 0 : iters;
  a.vy1 = wm - (gy0 + wm == R ? 0 : iters);
  a.vx0 = gx0 == 0 ? 0 : iters;
  a.vx1 = wn - (gx0 + wn == C ? 0 : iters);
  if (a.vy1 <= a.vy0 || a.vx1 <= a.vx0) return 0;
  a.cap_1 = coef[0];
  a.rx_1 = coef[1];
  a.ry_1 = coef[2];
  a.rz_1 = coef[3];
  a.amb = coef[4];
  if (hotspot_variant() == 4) {
    constexpr int RH = kV4V * kV4NWY, RW = 32 * kV4NWX;
    const int oty = RH - 2 * iters, otx = RW - 2 * iters;
    const int64_t gy4 = (a.vy1 - a.vy0 + oty - 1) / oty, gx4 = (a.vx1 - a.vx0 + otx - 1) / otx;
    if (gy4 > 65535) return fail(NU_EINVAL, "hotspot window too tall (%lld tile rows)", (long long)gy4);
    const int smem4 = 2 * (kV4NWY * kV4V / 2 + 2) * (RW + 2) * 8;
    cudaFuncSetAttribute(hotspot_kernel_v4<kV4V, kV4NWX, kV4NWY>,
                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem4);
    hotspot_kernel_v4<kV4V, kV4NWX, kV4NWY><<<dim3(static_cast<unsigned>(gx4), static_cast<unsigned>(gy4)),
                                             kV4NWX * kV4NWY * 32, smem4, stream>>>(a);
    count_launches(1);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? 0 : cuda_fail(e, "hotspot_kernel_v4 launch");
  }
  if (hotspot_variant() == 3) {
    constexpr int RH = kV3V * kV3NWY, RW = 32 * kV3NWX;
    const int oty = RH - 2 * iters, otx = RW - 2 * iters;
    const int64_t gy3 = (a.vy1 - a.vy0 + oty - 1) / oty, gx3 = (a.vx1 - a.vx0 + otx - 1) / otx;
    if (gy3 > 65535) return fail(NU_EINVAL, "hotspot window too tall (%lld tile rows)", (long long)gy3);
    const int smem3 = 2 * (RH + 2) * (RW + 2) * 4;
    cudaFuncSetAttribute(hotspot_kernel_v3<kV3V, kV3NWX, kV3NWY>,
                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem3);
    hotspot_kernel_v3<kV3V, kV3NWX, kV3NWY><<<dim3(static_cast<unsigned>(gx3), static_cast<unsigned>(gy3)),
                                             kV3NWX * kV3NWY * 32, smem3, stream>>>(a);
    count_launches(1);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? 0 : cuda_fail(e, "hotspot_kernel_v3 launch");
  }
  if (hotspot_variant() == 2) {
    const int oty = kRPT * kNWY - 2 * iters, otx = 32 * kNWX - 2 * iters;
    const int64_t gy2 = (a.vy1 - a.vy0 + oty - 1) / oty, gx2 = (a.vx1 - a.vx0 + otx - 1) / otx;
    if (gy2 > 65535) return fail(NU_EINVAL, "hotspot window too tall (%lld tile rows)", (long long)gy2);
    hotspot_kernel_v2<kRPT, kNWX, kNWY><<<dim3(static_cast<unsigned>(gx2), static_cast<unsigned>(gy2)),
                                          kNWX * kNWY * 32, 0, stream>>>(a);
    count_launches(1);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? 0 : cuda_fail(e, "hotspot_kernel_v2 launch");
  }
  const int64_t gy = (a.vy1 - a.vy0 + kTY - 1) / kTY, gx = (a.vx1 - a.vx0 + kTX - 1) / kTX;
  if (gy > 65535) return fail(NU_EINVAL, "hotspot window too tall (%lld tile rows)", (long long)gy);
  const size_t smem = 3ull * (kTY + 2 * iters) * (kTX + 2 * iters) * sizeof(float);
  // per device context; cheap next to a launch
  cudaFuncSetAttribute(hotspot_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       static_cast<int>(3ull * (kTY + 2 * kHotspotMaxIters) * (kTX + 2 * kHotspotMaxIters) * 4));
  hotspot_kernel<<<dim3(static_cast<unsigned>(gx), static_cast<unsigned>(gy)), dim3(kWX, kWY), smem, stream>>>(a);
  count_launches(1);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : cuda_fail(e, "hotspot_kernel launch");
}

}  // namespace nu
