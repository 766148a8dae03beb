// HotSpot-2D leaf (S§8(f) NEXT-3; §IV-B): the explicit
// thermal update of [18] (reading RH1, coefficients RH2) on a window
// of the grid resident in HBM, several iterations per launch.
//
// The paper's leaf loads a block and its borders into (block+2)^2 local-memory
// arrays and does one iteration.  Here a tile (128 x 132 cells, output
// 112 x 116 at 8 iterations) is loaded once, temperature is kept in registers
// and power in shared memory, and all `iters` iterations run on chip (the valid
// region shrinks by one cell per iteration on every side that is not a grid
// edge), so HBM is read once and written once per `iters` iterations.  The
// product kernel (hotspot_kernel_tma) is persistent and loads the next tile by
// TMA while the current one iterates; hotspot_kernel_v5 (128 x 96 tiles, plain
// loads) serves windows whose base or leading dimension is not 16-byte aligned.
//
// Arithmetic contract (RH4, revised): the update
//     T' = T + cap_1 (P + (S + N - 2T) ry_1 + (E + W - 2T) rx_1 + (amb - T) rz_1)
// is evaluated in the expanded form
//     T' = kt T + kx (E + W) + ky (S + N) + q,   q = cap_1 P + cap_1 rz_1 amb
// with kt = 1 - cap_1 (2 rx_1 + 2 ry_1 + rz_1), kx = cap_1 rx_1, ky = cap_1 ry_1
// (rounded to fp32 once on the host from the fp32 coefficients) and q
// computed once per cell and tile, q = fma(cap_1, P, kq).  Per cell update one
// fixed fp32 sequence (round-to-nearest, fma = one rounding):
//     u = fma(kt, t, q);  u = fma(kx, e + w, u);  t' = fma(ky, s + n, u)
// written with __fadd_rn/__fmaf_rn so the compiler cannot reassociate or
// re-fuse it: 2 FADD + 3 FFMA per update (the first form took 3 FADD + 6
// FFMA).  The weights kt, kx, kx, ky, ky are positive and sum to 1 - cap_1
// rz_1, so rounding errors do not grow (RH3's bound holds).  The result of a
// cell is independent of tiling, iterations per launch and launch order:
// in-HBM and out-of-core runs agree bit for bit, and so does an exact fp32
// emulation of this sequence.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include <algorithm>
#include <map>
#include <mutex>
#include <utility>

#include "leaf_common.cuh"
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
  float kt, kx, ky;          // expanded-form weights (see the contract above)
  float kc, kq;              // q = fma(kc, P, kq): kc = cap_1, kq = cap_1 rz_1 amb
};

// q = the update's constant part of one cell (P and the ambient term)
__device__ __forceinline__ float q_of(float p, const Args& a) { return __fmaf_rn(a.kc, p, a.kq); }

__device__ __forceinline__ float update(float t, float q, float n, float s, float e, float w,
                                        const Args& a) {
  float u = __fmaf_rn(a.kt, t, q);
  u = __fmaf_rn(a.kx, __fadd_rn(e, w), u);
  return __fmaf_rn(a.ky, __fadd_rn(s, n), u);
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
// Power row segment from shared memory.  volatile: read where written (one row
// ahead of its use), not hoisted into registers for all rows of the run.
__device__ __forceinline__ float4 ld_power(const float* q) {
  float4 p;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(p.x), "=f"(p.y), "=f"(p.z), "=f"(p.w)
               : "r"(static_cast<unsigned>(__cvta_generic_to_shared(q))));
  return p;
}

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

// NAMED: synchronise the NW compute warps on named barrier 1 instead of
// __syncthreads.  The halo buffer's parity continues from `k0` so consecutive
// iterations, also across tiles, never share a buffer.  (Waiting on the two
// vertical neighbours' mbarriers instead of a CTA-wide barrier was measured
// slower twice: waiting right after publishing, and split-phase — publish the
// run's first and last rows first, compute the interior, wait at the next
// iteration (1507 vs 1674 GCUPS): the mbarrier polling costs more issue slots
// than the barrier skew it removes.)
// qv: the lane's q per row in registers (the persistent kernel), else NULL and
// q is read from the shared-memory tile `ps` one row ahead (v5).
template <int V, int NW, bool EDGE, bool NAMED = false>
__device__ __forceinline__ void v5_iterate(const Args& a, float4 (&v)[V], const float* __restrict__ ps,
                                           float* __restrict__ hb, int lane, int warp, int rtop, int rbot,
                                           int cl, int cr, int k0 = 0, const float4* qv = nullptr) {
  constexpr int RW = 128;
  // The persistent kernel unrolls the iteration loop by two: the new rows then
  // alternate between two register sets instead of being moved back into the
  // loop-carried ones (26 moves per iteration; 1584 -> 1674 GCUPS).  v5 has no
  // registers to spare for it.
  constexpr int kUnroll = NAMED ? 2 : 1;
#pragma unroll kUnroll
  for (int k = 0; k < a.iters; ++k) {
    float* buf = hb + ((k0 + k) & 1) * (NW * 2 * RW);
    *reinterpret_cast<float4*>(buf + (warp * 2 + 0) * RW + 4 * lane) = v[0];        // my first row
    *reinterpret_cast<float4*>(buf + (warp * 2 + 1) * RW + 4 * lane) = v[V - 1];    // my last row
    if (NAMED)
      asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory");
    else
      __syncthreads();
    // The tile's top (bottom) warp reads its own row as the northern (southern)
    // neighbour: a select on the index, no branch.  Those rows lie in the
    // tile's recomputed margin (never written back) unless they are the grid
    // edge, where v5_row's clamp replaces the neighbour anyway.
    const int up = warp > 0 ? (warp - 1) * 2 + 1 : 0, dn = warp < NW - 1 ? (warp + 1) * 2 : (NW - 1) * 2 + 1;
    float4 prev = *reinterpret_cast<const float4*>(buf + up * RW + 4 * lane);
    const float4 below = *reinterpret_cast<const float4*>(buf + dn * RW + 4 * lane);
    // Row r's W/E shuffles and power load are issued one row ahead, so their
    // latency hides behind row r-1's arithmetic (4 warps per SM sub-partition
    // are too few to cover it otherwise).
    float wl_n = __shfl_up_sync(0xffffffffu, v[0].w, 1);
    float er_n = __shfl_down_sync(0xffffffffu, v[0].x, 1);
    float4 p_n = NAMED ? qv[0] : ld_power(ps + (warp * V) * RW + 4 * lane);
#pragma unroll
    for (int r = 0; r < V; ++r) {
      const float4 c = v[r];
      const float4 s = r < V - 1 ? v[r + 1] : below;
      const float wl = wl_n, er = er_n;
      const float4 p = p_n;
      if (r + 1 < V) {
        wl_n = __shfl_up_sync(0xffffffffu, v[r + 1].w, 1);
        er_n = __shfl_down_sync(0xffffffffu, v[r + 1].x, 1);
        p_n = NAMED ? qv[r + 1] : ld_power(ps + (warp * V + r + 1) * RW + 4 * lane);
      }
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
  float* ps = sm5;                 // q = fma(cap_1, power, kq) of the tile, RH x RW
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
    *reinterpret_cast<float4*>(ps + (r0 + r) * RW + x0) =
        make_float4(q_of(p[0], a), q_of(p[1], a), q_of(p[2], a), q_of(p[3], a));
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

// ---------------------------------------------------------------------------
// Persistent TMA leaf (the product kernel when the window's base and leading
// dimensions are 16-byte aligned): one CTA per SM claims tiles (128 columns x
// 128 rows, output 112 x 112 at 8 iterations) and runs them with 16 warps, 4
// per SM sub-partition; a lane owns 4 columns x 8 rows (the v5 scheme above)
// and keeps their temperature AND their q (RH4) in registers, so an
// update reads nothing from shared memory but the two halo rows per iteration
// (128 registers; measured 2379 GCUPS against 2330 for 12 warps x 10 rows, 2235
// for 16 x 7, 2219 for 8 x 15, and 2022 with q read from shared memory).
// Thread 0 also issues the loads.  While the warps iterate tile i, TMA brings
// tile i+1's temperature (single buffer, freed as soon as the compute warps
// have copied it into registers) and power (double buffer) into shared memory,
// so HBM traffic overlaps the arithmetic instead of alternating with it.
// Out-of-window cells are zero-filled by TMA, as v5's predicated loads do.
constexpr int kPW = 16, kPV = 8, kPRH = kPW * kPV, kPRW = 128;

// Tile t -> (tile row, tile column), row-major.  CTAs CLAIM tiles in this
// order from a counter (atomicAdd) instead of taking a static t = c, c + grid,
// ...: with a static walk, a tile row of grid / 2 tiles (or any width that
// makes grid ~ a multiple of it) hands one tile column to the same few CTAs,
// and a column of slower clamped tiles at the grid's west or east edge then
// stretches the whole launch (measured on the out-of-core plan's edge windows:
// 0.33 -> 0.52 ms per launch once a window shrinks to 74 tile columns, and a
// row skew only moved the resonance to 75 columns).
__device__ __forceinline__ void tile_of(int t, int tiles_x, int& by, int& bx) {
  by = t / tiles_x;
  bx = t - by * tiles_x;
}
constexpr int kPTileBytes = kPRH * kPRW * 4;                    // 64 KiB
constexpr int kPHaloFloats = 2 * kPW * 2 * kPRW;               // 32 KiB
constexpr int kPSmem = 3 * kPTileBytes + kPHaloFloats * 4 + 64;   // T | P[2] | halo | barriers, tile ids

__device__ __forceinline__ void tma_load_tile(uint32_t dst, const CUtensorMap* map, int x, int y, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(bar)
      : "memory");
}

__global__ void __launch_bounds__(kPW * 32, 1)
    hotspot_kernel_tma(const __grid_constant__ CUtensorMap mT, const __grid_constant__ CUtensorMap mP, Args a,
                       int tiles_x, int tiles, int rx0, int sx, bool vec_out, unsigned* ctr) {
  using namespace nu::leaf;
  extern __shared__ __align__(128) float smp[];
  float* tb = smp;                                   // temperature of the next tile
  float* pb = smp + kPRH * kPRW;                     // power, two tiles
  float* hb = smp + 3 * kPRH * kPRW;                 // halo rows
  uint64_t* bars = reinterpret_cast<uint64_t*>(hb + kPHaloFloats);
  const uint32_t full0 = smem_u32(bars), pempty0 = smem_u32(bars + 2), tempty = smem_u32(bars + 4);
  volatile int* tile_id = reinterpret_cast<volatile int*>(bars + 6);   // [j % 2]: tile of load j, -1 = none
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int h = a.iters, OTY = kPRH - 2 * h;
  // Thread 0 is also the producer: it issues tile j's two TMA loads (T into
  // the single T buffer, P into P buffer j % 2), both completing on full[j % 2].
  auto issue = [&](int j, int t) {
    int by, bx;
    tile_of(t, tiles_x, by, bx);
    const int ry = static_cast<int>(a.vy0) + by * OTY - h, rx = rx0 + bx * sx;
    const uint32_t fb = full0 + 8 * (j & 1);
    mbar_arrive_expect_tx(fb, 2 * kPTileBytes);
    tma_load_tile(smem_u32(tb), &mT, rx, ry, fb);
    tma_load_tile(smem_u32(pb + (j & 1) * kPRH * kPRW), &mP, rx, ry, fb);
  };
  if (threadIdx.x == 0) {
    mbar_init(full0, 1);
    mbar_init(full0 + 8, 1);
    mbar_init(pempty0, kPW);
    mbar_init(pempty0 + 8, kPW);
    mbar_init(tempty, kPW);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    prefetch_tmap(&mT);
    prefetch_tmap(&mP);
    const int t0 = static_cast<int>(atomicAdd(ctr, 1u));
    tile_id[0] = t0 < tiles ? t0 : -1;
    if (t0 < tiles) issue(0, t0);
    else mbar_arrive(full0);                     // nothing to load: release the consumers
  }
  __syncthreads();
  const int r0 = warp * kPV, x0 = 4 * lane;
  for (int i = 0;; ++i) {
    mbar_wait(full0 + 8 * (i & 1), (i >> 1) & 1);
    const int t = tile_id[i & 1];
    if (t < 0) break;
    int by, bx;
    tile_of(t, tiles_x, by, bx);
    const int64_t oy0 = a.vy0 + static_cast<int64_t>(by) * OTY;
    const int64_t ry = oy0 - h, rx = rx0 + static_cast<int64_t>(bx) * sx;
    float4 v[kPV];
#pragma unroll
    for (int r = 0; r < kPV; ++r) v[r] = *reinterpret_cast<const float4*>(tb + (r0 + r) * kPRW + x0);
    __syncwarp();
    if (lane == 0) mbar_arrive(tempty);
    if (threadIdx.x == 0) {
      const int tn = static_cast<int>(atomicAdd(ctr, 1u));
      if (tn < tiles) {
        mbar_wait(tempty, i & 1);                                      // every warp holds tile i's T
        if (i >= 1) mbar_wait(pempty0 + 8 * ((i + 1) & 1), ((i - 1) >> 1) & 1);   // tile i-1 done with its P
        tile_id[(i + 1) & 1] = tn;
        issue(i + 1, tn);
      } else {
        tile_id[(i + 1) & 1] = -1;
        mbar_arrive(full0 + 8 * ((i + 1) & 1));
      }
    }
    __syncwarp();
    // power -> q of this lane's own cells (the only ones it reads back), in
    // place; the fence orders these generic writes before the TMA that will
    // refill the buffer once every warp has released it (pempty)
    const float* ps = pb + (i & 1) * kPRH * kPRW;
    float4 qv[kPV];
#pragma unroll
    for (int r = 0; r < kPV; ++r) {
      const float4 pv = ld_power(ps + (r0 + r) * kPRW + x0);
      qv[r] = make_float4(q_of(pv.x, a), q_of(pv.y, a), q_of(pv.z, a), q_of(pv.w, a));
    }
    const int64_t gy_top = a.gy0 + ry, gx_left = a.gx0 + rx;
    const bool edge = gy_top <= 0 || gy_top + kPRH >= a.R || gx_left <= 0 || gx_left + kPRW >= a.C;
    if (edge) {
      const int64_t gx = gx_left + x0;
      const int cl = (gx <= 0 && gx > -4) ? static_cast<int>(-gx) : -1;
      const int cr = (a.C - 1 - gx >= 0 && a.C - 1 - gx < 4) ? static_cast<int>(a.C - 1 - gx) : -1;
      const int64_t gy = gy_top + r0;
      const int rtop = (gy <= 0 && gy > -kPV) ? static_cast<int>(-gy) : -1;
      const int rbot = (a.R - 1 - gy >= 0 && a.R - 1 - gy < kPV) ? static_cast<int>(a.R - 1 - gy) : -1;
      v5_iterate<kPV, kPW, true, true>(a, v, ps, hb, lane, warp, rtop, rbot, cl, cr, i * h, qv);
    } else {
      v5_iterate<kPV, kPW, false, true>(a, v, ps, hb, lane, warp, -1, -1, -1, -1, i * h, qv);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(pempty0 + 8 * (i & 1));
    const int64_t ylo = max(oy0, a.vy0), yhi = min(oy0 + OTY, a.vy1);
    const int64_t xlo = max(rx + h, a.vx0), xhi = min(rx + h + sx, a.vx1);
    const int64_t wx = rx + x0;
    const bool full4 = vec_out && wx >= xlo && wx + 4 <= xhi;    // 16-B aligned: rx, ldo, tout
    float* orow = a.tout + (ry + r0) * a.ldo + wx;
#pragma unroll
    for (int r = 0; r < kPV; ++r, orow += a.ldo) {
      const int64_t wy = ry + r0 + r;
      if (wy < ylo || wy >= yhi) continue;
      if (full4) {
        *reinterpret_cast<float4*>(orow) = v[r];
      } else {
        const float tv[4] = {v[r].x, v[r].y, v[r].z, v[r].w};
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (wx + j >= xlo && wx + j < xhi) orow[j] = tv[j];
      }
    }
  }
  // Every CTA made exactly one failing claim before leaving; the last one out
  // re-arms the counter for the next launch on this stream.
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(ctr + 1, 1u) == gridDim.x - 1) {
      ctr[0] = 0;
      ctr[1] = 0;
    }
  }
}

constexpr int kV5V = 12, kV5NW = 8;   // V rows per thread (registers), NW warps per CTA

// Tile counters of the persistent kernel, one pair per (device, stream): a
// launch claims tiles from its stream's counter and its last CTA resets it, so
// launches on one stream (which never overlap) can share it, and launches on
// different streams (virtual siblings on one device run concurrently) never do.
static unsigned* tile_counter(int dev, cudaStream_t s) {
  static std::mutex m;
  static std::map<std::pair<int, cudaStream_t>, unsigned*> ctrs;
  std::lock_guard<std::mutex> g(m);
  auto it = ctrs.find({dev, s});
  if (it != ctrs.end()) return it->second;
  unsigned* p = nullptr;
  if (cudaMalloc(&p, 2 * sizeof(unsigned)) != cudaSuccess) return nullptr;
  if (cudaMemset(p, 0, 2 * sizeof(unsigned)) != cudaSuccess) {
    cudaFree(p);
    return nullptr;
  }
  ctrs[{dev, s}] = p;
  return p;
}

}  // namespace hs

int hotspot_max_iters_per_launch() { return kHotspotMaxIters; }

void hotspot_preload() {
  using namespace hs;
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, hotspot_kernel_v5<kV5V, kV5NW>);
  cudaFuncGetAttributes(&fa, hotspot_kernel_tma);
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
  // expanded-form weights, each rounded once from the fp32 coefficients (RH4)
  const double cap = coef[0], rx = coef[1], ry = coef[2], rz = coef[3], amb = coef[4];
  a.kt = static_cast<float>(1.0 - cap * (2.0 * rx + 2.0 * ry + rz));
  a.kx = static_cast<float>(cap * rx);
  a.ky = static_cast<float>(cap * ry);
  a.kc = coef[0];
  a.kq = static_cast<float>(cap * rz * amb);
  const bool aligned = (reinterpret_cast<uintptr_t>(tin) & 15) == 0 && (reinterpret_cast<uintptr_t>(pw) & 15) == 0 &&
                       ldt % 4 == 0 && ldp % 4 == 0 && wm < (1ll << 30) && wn < (1ll << 30);
  if (aligned) {
    CUtensorMap mT, mP;
    int rc = leaf::encode_2d(&mT, tin, wn, wm, ldt, kPRW, kPRH, CU_TENSOR_MAP_SWIZZLE_NONE);
    if (!rc) rc = leaf::encode_2d(&mP, pw, wn, wm, ldp, kPRW, kPRH, CU_TENSOR_MAP_SWIZZLE_NONE);
    if (rc) return rc;
    // TMA reads a box whose first column is 16-byte aligned: tiles start at
    // multiples of 4 columns and advance by sx (a multiple of 4, <= 128 - 2h)
    // output columns; tile b owns [rx0 + b sx + h, rx0 + (b + 1) sx + h).
    const int oty = kPRH - 2 * iters, sx = (kPRW - 2 * iters) / 4 * 4;
    const int64_t rx0 = (a.vx0 - iters) >= 0 ? (a.vx0 - iters) / 4 * 4 : -((iters - a.vx0 + 3) / 4 * 4);
    const int64_t ty = (a.vy1 - a.vy0 + oty - 1) / oty, tx = (a.vx1 - (rx0 + iters) + sx - 1) / sx;
    if (ty * tx >= (1ll << 31)) return fail(NU_EINVAL, "hotspot window too large");
    int dev = 0;
    cudaGetDevice(&dev);
    const int tiles = static_cast<int>(ty * tx);
    const int grid = std::min(tiles, sms_of(dev));
    unsigned* ctr = tile_counter(dev, stream);
    if (!ctr) return fail(NU_ECUDA, "hotspot: tile counter allocation failed");
    cudaFuncSetAttribute(hotspot_kernel_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, kPSmem);
    hotspot_kernel_tma<<<grid, kPW * 32, kPSmem, stream>>>(mT, mP, a, static_cast<int>(tx), tiles,
                                                                   static_cast<int>(rx0), sx,
                                                                   (reinterpret_cast<uintptr_t>(tout) & 15) == 0 && ldo % 4 == 0, ctr);
    count_launches(1);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? 0 : cuda_fail(e, "hotspot_kernel_tma launch");
  }
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
