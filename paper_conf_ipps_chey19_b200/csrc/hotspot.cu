// HotSpot-2D leaf (S§8(f) NEXT-3; §IV-B): the explicit
// thermal update of [18] (reading RH1, coefficients RH2) on a window
// of the grid resident in HBM, several iterations per launch.
//
// The paper's leaf loads a block and its borders into (block+2)^2 local-memory
// arrays and does one iteration.  Here a CTA loads its tile (128
// columns x 96 rows, output 112 x 80 at 8 iterations) once, keeps temperature
// in registers and power in shared memory, and performs all `iters`
// iterations on chip (the valid region shrinks by one cell per iteration on
// every side that is not a grid edge), so HBM is read once and written once
// per `iters` iterations.
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

// ---------------------------------------------------------------------------
// v5: a lane owns 4 consecutive columns x V rows in registers, a warp spans
// the CTA tile's 128 columns, NW warps stack vertically (tile 128 x NW*V).
// Per iteration: W/E neighbours of the lane's outer columns come from the
// adjacent lanes (one shfl.up + one shfl.down per row of 4 cells, inner
// columns from registers), N/S neighbours from registers inside the run and,
// for the run's first / last row, from the vertically adjacent warps through
// a double-buffered shared-memory row (one barrier per iteration); power lives
// in shared memory (one 16-byte load per row of 4 cells).  Same RH4 sequence
// per cell, so v5 is bitwise equal to the fp32 emulation (and to the
// round-1 leaves v1-v4, replaced by this one: DESIGN.md §11).
template <bool EDGE>
__device__ __forceinline__ float4 v5_row(const float4 c, const float4 p, const float4 n, const float4 s, float wl,
                                         float er, const Args& a, bool rtop, bool rbot, int cl, int cr) {
  float nn[4] = {n.x, n.y, n.z, n.w}, ss[4] = {s.x, s.y, s.z, s.w};
  const float cc[4] = {c.x, c.y, c.z, c.w}, pp[4] = {p.x, p.y, p.z, p.w};
  float out[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    float w = j > 0 ? cc[j - 1] : wl;
    float e = j < 3 ? cc[j + 1] : er;
    float nj = nn[j], sj = ss[j];
    if (EDGE) {
      if (rtop) nj = cc[j];
      if (rbot) sj = cc[j];
      if (j == cl) w = cc[j];
      if (j == cr) e = cc[j];
    }
    out[j] = update(cc[j], pp[j], nj, sj, e, w, a);
  }
  return make_float4(out[0], out[1], out[2], out[3]);
}

template <int V, int NW, bool EDGE>
__device__ __forceinline__ void v5_iterate(const Args& a, float4 (&v)[V], const float* __restrict__ ps,
                                           float* __restrict__ hb, int lane, int warp, int rtop, int rbot,
                                           int cl, int cr) {
  constexpr int RW = 128;
  for (int k = 0; k < a.iters; ++k) {
    float* buf = hb + (k & 1) * (NW * 2 * RW);
    *reinterpret_cast<float4*>(buf + (warp * 2 + 0) * RW + 4 * lane) = v[0];        // my first row
    *reinterpret_cast<float4*>(buf + (warp * 2 + 1) * RW + 4 * lane) = v[V - 1];    // my last row
    __syncthreads();
    float4 prev = warp > 0 ? *reinterpret_cast<const float4*>(buf + ((warp - 1) * 2 + 1) * RW + 4 * lane) : v[0];
    const float4 below =
        warp < NW - 1 ? *reinterpret_cast<const float4*>(buf + ((warp + 1) * 2 + 0) * RW + 4 * lane) : v[V - 1];
#pragma unroll
    for (int r = 0; r < V; ++r) {
      const float4 c = v[r];
      const float4 s = r < V - 1 ? v[r + 1] : below;
      const float wl = __shfl_up_sync(0xffffffffu, c.w, 1);
      const float er = __shfl_down_sync(0xffffffffu, c.x, 1);
      float4 p;   // volatile: read per row, not hoisted into registers for all V rows
      asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                   : "=f"(p.x), "=f"(p.y), "=f"(p.z), "=f"(p.w)
                   : "r"(static_cast<unsigned>(__cvta_generic_to_shared(ps + (warp * V + r) * RW + 4 * lane))));
      v[r] = v5_row<EDGE>(c, p, prev, s, wl, er, a, EDGE && r == rtop, EDGE && r == rbot, cl, cr);
      prev = c;
    }
  }
}

// 2 CTAs per SM (128 registers): one CTA's loads overlap the other's iterations.
template <int V, int NW>
__global__ void __launch_bounds__(NW * 32, 2) hotspot_kernel_v5(Args a) {
  constexpr int RW = 128, RH = NW * V;
  extern __shared__ float sm5[];
  float* ps = sm5;                 // power tile RH x RW
  float* hb = sm5 + RH * RW;       // 2 parities x NW warps x {first, last} row x RW
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int h = a.iters;
  const int OTY = RH - 2 * h, OTX = RW - 2 * h;
  const int64_t oy0 = a.vy0 + static_cast<int64_t>(blockIdx.y) * OTY;
  const int64_t ox0 = a.vx0 + static_cast<int64_t>(blockIdx.x) * OTX;
  const int64_t ry = oy0 - h, rx = ox0 - h;        // tile origin (window coordinates)
  const int r0 = warp * V, x0 = 4 * lane;
  float4 v[V];
#pragma unroll
  for (int r = 0; r < V; ++r) {
    const int64_t wy = ry + r0 + r;
    const bool yin = wy >= 0 && wy < a.wm;
    float t[4], p[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int64_t wx = rx + x0 + j;
      const bool in = yin && wx >= 0 && wx < a.wn;
      t[j] = in ? __ldg(a.tin + wy * a.ldt + wx) : 0.0f;
      p[j] = in ? __ldg(a.pw + wy * a.ldp + wx) : 0.0f;
    }
    v[r] = make_float4(t[0], t[1], t[2], t[3]);
    *reinterpret_cast<float4*>(ps + (r0 + r) * RW + x0) = make_float4(p[0], p[1], p[2], p[3]);
  }
  // (the first iteration's barrier also orders these power stores)
  const int64_t gy_top = a.gy0 + ry, gx_left = a.gx0 + rx;
  const bool edge = gy_top <= 0 || gy_top + RH >= a.R || gx_left <= 0 || gx_left + RW >= a.C;
  if (edge) {
    const int64_t gx = gx_left + x0;   // grid column of this lane's first cell
    const int cl = (gx <= 0 && gx > -4) ? static_cast<int>(-gx) : -1;
    const int cr = (a.C - 1 - gx >= 0 && a.C - 1 - gx < 4) ? static_cast<int>(a.C - 1 - gx) : -1;
    const int64_t gy = gy_top + r0;    // grid row of this thread's first cell
    const int rtop = (gy <= 0 && gy > -V) ? static_cast<int>(-gy) : -1;
    const int rbot = (a.R - 1 - gy >= 0 && a.R - 1 - gy < V) ? static_cast<int>(a.R - 1 - gy) : -1;
    v5_iterate<V, NW, true>(a, v, ps, hb, lane, warp, rtop, rbot, cl, cr);
  } else {
    v5_iterate<V, NW, false>(a, v, ps, hb, lane, warp, -1, -1, -1, -1);
  }
  const int64_t oy = oy0, ox = ox0;
  const int64_t ylo = max(oy, a.vy0), yhi = min(oy + OTY, a.vy1);
  const int64_t xlo = max(ox, a.vx0), xhi = min(ox + OTX, a.vx1);
#pragma unroll
  for (int r = 0; r < V; ++r) {
    const int64_t wy = ry + r0 + r;
    if (wy < ylo || wy >= yhi) continue;
    const float t[4] = {v[r].x, v[r].y, v[r].z, v[r].w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int64_t wx = rx + x0 + j;
      if (wx >= xlo && wx < xhi) a.tout[wy * a.ldo + wx] = t[j];
    }
  }
}

constexpr int kV5V = 12, kV5NW = 8;   // V rows per thread (registers), NW warps per CTA

}  // namespace hs

int hotspot_max_iters_per_launch() { return kHotspotMaxIters; }

void hotspot_preload() {
  using namespace hs;
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, hotspot_kernel_v5<kV5V, kV5NW>);
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
  {
    constexpr int RH = kV5V * kV5NW, RW = 128;
    const int oty = RH - 2 * iters, otx = RW - 2 * iters;
    const int64_t gy5 = (a.vy1 - a.vy0 + oty - 1) / oty, gx5 = (a.vx1 - a.vx0 + otx - 1) / otx;
    if (gy5 > 65535) return fail(NU_EINVAL, "hotspot window too tall (%lld tile rows)", (long long)gy5);
    const int smem5 = (RH * RW + 2 * kV5NW * 2 * RW) * 4;
    cudaFuncSetAttribute(hotspot_kernel_v5<kV5V, kV5NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem5);
    hotspot_kernel_v5<kV5V, kV5NW><<<dim3(static_cast<unsigned>(gx5), static_cast<unsigned>(gy5)), kV5NW * 32,
                                     smem5, stream>>>(a);
    count_launches(1);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? 0 : cuda_fail(e, "hotspot_kernel_v5 launch");
  }
}

}  // namespace nu
