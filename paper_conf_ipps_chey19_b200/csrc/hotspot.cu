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
// Arithmetic contract: every cell update is
//     t + cap_1 * (((p + ((s + n) - 2t) * ry_1) + ((e + w) - 2t) * rx_1) + (amb - t) * rz_1)
// evaluated left to right in fp32 with round-to-nearest and no FMA
// contraction (__fadd_rn/__fmul_rn), so the result of a cell is independent
// of tiling, iterations per launch and launch order: in-HBM and out-of-core
// runs agree bit for bit, and so does an fp32 numpy emulation of the update.
#include <cuda_runtime.h>
#include <stdint.h>

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
  const float two_t = __fmul_rn(2.0f, t);
  const float ly = __fmul_rn(__fsub_rn(__fadd_rn(s, n), two_t), a.ry_1);
  const float lx = __fmul_rn(__fsub_rn(__fadd_rn(e, w), two_t), a.rx_1);
  const float lz = __fmul_rn(__fsub_rn(a.amb, t), a.rz_1);
  const float d = __fadd_rn(__fadd_rn(__fadd_rn(p, ly), lx), lz);
  return __fadd_rn(t, __fmul_rn(a.cap_1, d));
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

  // data_down HBM -> SMEM: the tile with its borders (coalesced rows)
  for (int y = ty; y < hy; y += kWY) {
    const float* trow = a.tin + (sy0 + y) * a.ldt + sx0;
    const float* prow = a.pw + (sy0 + y) * a.ldp + sx0;
    for (int x = tx; x < hx; x += kWX) {
      cur[y * SX + x] = __ldg(trow + x);
      pwr[y * SX + x] = __ldg(prow + x);
    }
  }
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

}  // namespace hs

int hotspot_max_iters_per_launch() { return kHotspotMaxIters; }

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
  const int64_t gy = (a.vy1 - a.vy0 + kTY - 1) / kTY, gx = (a.vx1 - a.vx0 + kTX - 1) / kTX;
  if (gy > 65535) return fail(NU_EINVAL, "hotspot window too tall (%lld tile rows)", (long long)gy);
  const size_t smem = 3ull * (kTY + 2 * iters) * (kTX + 2 * iters) * sizeof(float);
  // per device context; cheap next to a launch
  cudaFuncSetAttribute(hotspot_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       static_cast<int>(3ull * (kTY + 2 * kHotspotMaxIters) * (kTX + 2 * kHotspotMaxIters) * 4));
  hotspot_kernel<<<dim3(static_cast<unsigned>(gx), static_cast<unsigned>(gy)), dim3(kWX, kWY), smem, stream>>>(a);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : cuda_fail(e, "hotspot_kernel launch");
}

}  // namespace nu
