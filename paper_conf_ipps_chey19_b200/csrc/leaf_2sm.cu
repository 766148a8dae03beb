// Leaf kernel v1: a CTA pair (thread-block cluster of 2 on one TPC) computes
// a 256 x 256 tile of C with tcgen05.mma.cta_group::2 (UMMA M = 256).
//
// Same contract and arithmetic as v0 (leaf_sm100.cu: 3xTF32, TMEM
// accumulation per k_chunk, fp32 RN epilogue add), but each CTA stages only
// its half of the operands: CTA r holds A rows [r*128, r*128+128) and B
// columns [r*128, r*128+128) of the pair tile.  The leader CTA (rank 0)
// issues the MMAs, which read both CTAs' shared memory, so each SM's shared
// memory supplies 8 KiB per k8 step instead of 12 KiB.
//
// The tensor core truncates the low 13 mantissa bits of an fp32 operand fed
// as tf32 (probed on the box: tools/debug_leaf.py, R19), so the raw
// TMA tile IS the hi operand; the split only writes lo = x - trunc(x).  Raw
// tiles live in an RS-deep ring, lo tiles in an LS-deep ring.  Per k8 step
// the three MMAs run as (hi.lo, hi.hi, lo.hi) with the A collector keeping
// A_hi between the first two (one A read saved).
//
// Synchronisation across the pair:
//   full[s]    (each CTA)  own TMA bytes landed               -> own split warps
//   rempty[s]  (each CTA)  leader's commit, multicast          -> own TMA producer
//   xform[j]   (leader)    both CTAs' lo tile written (cnt 2)  -> MMA issuer
//   lempty[j]  (each CTA)  leader's commit, multicast          -> own split warps
//   tfull[a]   (each CTA)  leader's commit, multicast          -> own epilogue
//   tempty[a]  (leader)    both CTAs drained TMEM (count 2)    -> MMA issuer
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "leaf_2sm_common.cuh"
#include "leaf_common.cuh"
#include "northup_internal.h"

namespace nu {
namespace leaf {
namespace sm2 {

constexpr int BM = 256;                            // pair tile rows (UMMA M)
constexpr int BN = 256;                            // pair tile cols (UMMA N)
constexpr int BM_CTA = 128;                        // rows of A per CTA
constexpr int BN_CTA = 128;                        // cols of B per CTA
#ifndef NU_LEAF_RS
#define NU_LEAF_RS 4
#endif
#ifndef NU_LEAF_LS
#define NU_LEAF_LS 3
#endif
constexpr int RS = NU_LEAF_RS;                     // raw (TMA) ring depth
constexpr int LS = NU_LEAF_LS;                     // lo (split) ring depth
constexpr int A_BYTES = BM_CTA * BK * 4;           // 16 KiB
constexpr int B_BYTES = BN_CTA * BK * 4;           // 16 KiB
constexpr int TMA_BYTES = A_BYTES + B_BYTES;       // per CTA per stage
constexpr int STAGE_BYTES = TMA_BYTES;             // one raw or one lo stage
constexpr int XA_BYTES = BM_CTA * 2 * BK * 2;      // A' (bf16, 2 x BK virtual k): 16 KiB
#ifndef NU_LEAF_XFORM_WARPS
#define NU_LEAF_XFORM_WARPS 8
#endif
constexpr int XFORM_WARPS = NU_LEAF_XFORM_WARPS;   // split warps (2 .. 2+XFORM_WARPS-1)
constexpr int XFORM_THREADS = 32 * XFORM_WARPS;
constexpr int EPI_WARP0 = 2 + XFORM_WARPS;         // 4 epilogue warps follow
constexpr int EPI_THREADS = 128;
constexpr int NUM_THREADS = 32 * (EPI_WARP0 + 4);
constexpr int TMEM_COLS = 512;                     // 2 accumulators x 256 columns
constexpr int BAR_BYTES = 256;
constexpr int SMEM_BYTES = (RS + LS) * STAGE_BYTES + BAR_BYTES + 1024;
static_assert(SMEM_BYTES <= 227 * 1024, "shared memory budget");

// NU_LEAF2_PRESPLIT (build-time experiment, npass 2 only): a pre-pass writes the
// bf16 operands A' (M x 2K8, per k8 group [hi of 8 k | lo of 8 k]) and B'
// (2K8 x N, per k8 group [lo rows; hi rows]) to HBM once, and the producer
// TMA-loads them straight into the lo ring in the layouts the split warps
// would have written (SW128 K-major A', SW128 MN-major B'); the split warps
// only forward the barriers.
#ifndef NU_LEAF2_PRESPLIT
#define NU_LEAF2_PRESPLIT 0
#endif
__global__ void presplit_a_kernel(const float* __restrict__ A, int64_t lda, int M, int K, int K8,
                                  __nv_bfloat16* __restrict__ Ap) {
  const int64_t n = static_cast<int64_t>(M) * K8;
  for (int64_t idx = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; idx < n;
       idx += static_cast<int64_t>(gridDim.x) * blockDim.x) {
    const int64_t i = idx / K8;
    const int k = static_cast<int>(idx - i * K8);
    const float f = k < K ? A[i * lda + k] : 0.0f;
    const float h = trunc13(f);
    const int64_t o = i * 2 * K8 + 16 * (k >> 3) + (k & 7);
    Ap[o] = __float2bfloat16_rn(h);
    Ap[o + 8] = __float2bfloat16_rn(f - h);
  }
}
__global__ void presplit_b_kernel(const float* __restrict__ B, int64_t ldb, int K, int N, int K8,
                                  __nv_bfloat16* __restrict__ Bp) {
  const int64_t n = static_cast<int64_t>(K8) * N;
  for (int64_t idx = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; idx < n;
       idx += static_cast<int64_t>(gridDim.x) * blockDim.x) {
    const int k = static_cast<int>(idx / N);
    const int64_t j = idx - static_cast<int64_t>(k) * N;
    const float f = k < K ? B[static_cast<int64_t>(k) * ldb + j] : 0.0f;
    const float h = trunc13(f);
    const int64_t v = 16 * (k >> 3) + (k & 7);
    Bp[v * N + j] = __float2bfloat16_rn(f - h);
    Bp[(v + 8) * N + j] = __float2bfloat16_rn(h);
  }
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(NUM_THREADS, 1)
    leaf_gemm_2sm_kernel(const __grid_constant__ CUtensorMap tmA,
                         const __grid_constant__ CUtensorMap tmB, const Params p
#if NU_LEAF2_PRESPLIT
                         , const __grid_constant__ CUtensorMap tmAp, const __grid_constant__ CUtensorMap tmBp
#endif
                         ) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  uint8_t* raw_base = smem;                          // RS raw stages
  uint8_t* lo_base = smem + RS * STAGE_BYTES;         // LS lo stages
  uint8_t* bars = smem + (RS + LS) * STAGE_BYTES;
  const uint32_t bar_full = smem_u32(bars);
  const uint32_t bar_rempty = bar_full + 8 * RS;
  const uint32_t bar_xform = bar_rempty + 8 * RS;
  const uint32_t bar_lempty = bar_xform + 8 * LS;
  const uint32_t bar_tfull = bar_lempty + 8 * LS;
  const uint32_t bar_tempty = bar_tfull + 16;
  const uint32_t bar_rawfull = bar_tempty + 16;      // [RS] leader: both CTAs' raw tiles landed
#if NU_LEAF2_PRESPLIT
  const uint32_t bar_lofull = bar_rawfull + 8 * RS;  // [LS] the pre-split A'/B' tiles landed
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 8 * (3 * RS + 3 * LS + 4));
#else
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 8 * (3 * RS + 2 * LS + 4));
#endif

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;

  if (threadIdx.x == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < RS; ++s) {
      mbar_init(bar_full + 8 * s, 1);
      mbar_init(bar_rempty + 8 * s, 1);
      mbar_init(bar_rawfull + 8 * s, 2);   // one forwarded arrive per CTA
    }
    for (int j = 0; j < LS; ++j) {
      mbar_init(bar_xform + 8 * j, 2);   // one elected arrive per CTA
      mbar_init(bar_lempty + 8 * j, 1);
#if NU_LEAF2_PRESPLIT
      mbar_init(bar_lofull + 8 * j, 1);
#endif
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(bar_tfull + 8 * a, 1);
      mbar_init(bar_tempty + 8 * a, 2 * EPI_THREADS);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "n"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  const int cid = blockIdx.x >> 1;
  const int nclusters = gridDim.x >> 1;
  const int num_tiles = p.tiles_m * p.tiles_n;
  const int nkb = (p.K + BK - 1) / BK;
  const int nchunks = (nkb + p.kb_per_chunk - 1) / p.kb_per_chunk;

  if (warp == 0) {
    // ------------------------------------------------------ TMA producer (own half)
    if (lane == 0) {
      uint32_t it = 0;
      for (int t = cid; t < num_tiles; t += nclusters) {
        int mb, nb;
        tile_coords(t, p.tiles_m, p.tiles_n, p.band, mb, nb);
        const int row0 = mb * BM + rank * BM_CTA;
        const int col0 = nb * BN + rank * BN_CTA;
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const uint32_t s = it % RS, use = it / RS;
          mbar_wait(bar_rempty + 8 * s, (use & 1) ^ 1);
          const uint32_t full = bar_full + 8 * s;
          mbar_arrive_expect_tx(full, TMA_BYTES);
          const uint32_t sa = smem_u32(raw_base + s * STAGE_BYTES);
          const uint32_t sb = sa + A_BYTES;
          tma_load_2d(sa, &tmA, full, kb * BK, row0);
#pragma unroll
          for (int c = 0; c < BN_CTA / B_CHUNK; ++c)
            tma_load_2d(sb + c * B_CHUNK_BYTES, &tmB, full, col0 + c * B_CHUNK, kb * BK);
#if NU_LEAF2_PRESPLIT
          {
            const uint32_t j = it % LS, juse = it / LS;
            mbar_wait(bar_lempty + 8 * j, (juse & 1) ^ 1);
            const uint32_t lf = bar_lofull + 8 * j;
            mbar_arrive_expect_tx(lf, STAGE_BYTES);
            const uint32_t sl = smem_u32(lo_base + j * STAGE_BYTES);
            tma_load_2d(sl, &tmAp, lf, kb * 2 * BK, row0);                 // A': 64 virtual k x 128 rows
            tma_load_2d(sl + XA_BYTES, &tmBp, lf, col0, kb * 2 * BK);      // B': 64 n x 64 virtual k
            tma_load_2d(sl + XA_BYTES + 8192, &tmBp, lf, col0 + 64, kb * 2 * BK);
          }
#endif
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer (leader CTA only)
    if (leader && lane == 0) {
      const uint32_t idesc = idesc_tf32(BM, BN, 1u);
      const uint32_t idesc_bf = idesc_bf16(BM, BN);
      uint32_t it = 0, chunk_it = 0;
      long long w_xf = 0, w_te = 0, t_beg = clock64();   // profile mode (p.dbg)
      for (int t = cid; t < num_tiles; t += nclusters) {
        for (int ch = 0; ch < nchunks; ++ch, ++chunk_it) {
          const uint32_t acc = chunk_it & 1, ause = chunk_it >> 1;
          long long c0 = clock64();
          mbar_wait_cluster(bar_tempty + 8 * acc, (ause & 1) ^ 1);
          w_te += clock64() - c0;
          tc_fence_after();
          const uint32_t tmem_d = tmem_base + acc * BN;
          const int kb0 = ch * p.kb_per_chunk;
          const int kb1 = min(nkb, kb0 + p.kb_per_chunk);
          for (int kb = kb0; kb < kb1; ++kb, ++it) {
            const uint32_t s = it % RS, suse = it / RS;
            const uint32_t j = it % LS, juse = it / LS;
            const uint32_t a_hi = smem_u32(raw_base + s * STAGE_BYTES);
            const uint32_t b_hi = a_hi + A_BYTES;
            const uint32_t a_lo = smem_u32(lo_base + j * STAGE_BYTES);
            const uint32_t b_lo = a_lo + A_BYTES;
            if (p.npass == 2) {
              // hi.hi needs only the raw tiles: issue it as soon as both CTAs'
              // TMA landed, so the tensor core works while the split finishes
              // (R21); then both cross terms per k8 from the split's bf16 tiles.
              c0 = clock64();
              mbar_wait_cluster(bar_rawfull + 8 * s, suse & 1);
              w_xf += clock64() - c0;
              tc_fence_after();
#pragma unroll
              for (int k = 0; k < BK / UMMA_K; ++k)
                umma_tf32_2sm(tmem_d, umma_desc(a_hi + k * 32, 16, 1024),
                              umma_desc(b_hi + k * 1024, B_CHUNK_BYTES, 512, LAYOUT_SW128_BASE32B),
                              idesc, (kb == kb0 && k == 0) ? 0u : 1u);
              c0 = clock64();
              mbar_wait_cluster(bar_xform + 8 * j, juse & 1);
              w_xf += clock64() - c0;
              tc_fence_after();
#pragma unroll
              for (int k = 0; k < BK / UMMA_K; ++k)
                umma_bf16_2sm(tmem_d, umma_desc(a_lo + k * 32, 16, 1024),
                              umma_desc(a_lo + XA_BYTES + k * 2048, 8192, 1024), idesc_bf, 1u);
              umma_commit_pair(bar_rempty + 8 * s);
              umma_commit_pair(bar_lempty + 8 * j);
              continue;
            }
            c0 = clock64();
            if (!(p.b_kmajor & 1)) mbar_wait_cluster(bar_xform + 8 * j, juse & 1);   // exp. 1: no wait
            w_xf += clock64() - c0;
            tc_fence_after();
#pragma unroll
            for (int k = 0; k < BK / UMMA_K; ++k) {
              const uint64_t dah = umma_desc(a_hi + k * 32, 16, 1024);
              const uint64_t dal = umma_desc(a_lo + k * 32, 16, 1024);
              const uint64_t dbh = umma_desc(b_hi + k * 1024, B_CHUNK_BYTES, 512, LAYOUT_SW128_BASE32B);
              const uint64_t dbl = umma_desc(b_lo + k * 1024, B_CHUNK_BYTES, 512, LAYOUT_SW128_BASE32B);
              const uint32_t first = (kb == kb0 && k == 0) ? 0u : 1u;
              if (p.npass == 3) {
                umma_tf32_2sm_afill(tmem_d, dah, dbl, idesc, first);
                umma_tf32_2sm_alast(tmem_d, dah, dbh, idesc, 1u);
                umma_tf32_2sm(tmem_d, dal, dbh, idesc, 1u);
              } else {
                umma_tf32_2sm(tmem_d, dah, dbh, idesc, first);
              }
            }
            umma_commit_pair(bar_rempty + 8 * s);
            umma_commit_pair(bar_lempty + 8 * j);
          }
          umma_commit_pair(bar_tfull + 8 * acc);
        }
      }
      if (p.dbg) {
        float* d = p.dbg + 8 * cid;
        d[0] = static_cast<float>(clock64() - t_beg);
        d[1] = static_cast<float>(w_xf);
        d[2] = static_cast<float>(w_te);
        d[3] = static_cast<float>(it);
      }
    }
  } else if (warp < EPI_WARP0) {
    // ---------------------------------------------------- transform (own half)
    const int tid = threadIdx.x - 64;
    const uint32_t xform_leader0 = mapa(bar_xform, 0);
    const uint32_t rawfull_leader0 = mapa(bar_rawfull, 0);
    uint32_t it = 0;
    long long w_full = 0, w_lem = 0;
    for (int t = cid; t < num_tiles; t += nclusters) {
      for (int kb = 0; kb < nkb; ++kb, ++it) {
        const uint32_t s = it % RS, use = it / RS;
        const uint32_t j = it % LS, juse = it / LS;
        long long c0 = clock64();
        mbar_wait(bar_full + 8 * s, use & 1);
        if (p.npass == 2 && tid == 0) mbar_arrive_cluster(rawfull_leader0 + 8 * s);
#if NU_LEAF2_PRESPLIT
        mbar_wait(bar_lofull + 8 * j, juse & 1);
        if (tid == 0) mbar_arrive_cluster(xform_leader0 + 8 * j);
        w_full += clock64() - c0;
        continue;
#endif
        long long c1 = clock64();
        mbar_wait(bar_lempty + 8 * j, (juse & 1) ^ 1);
        w_full += c1 - c0;
        w_lem += clock64() - c1;
        const uint32_t raw = smem_u32(raw_base + s * STAGE_BYTES);
        const uint32_t lo = smem_u32(lo_base + j * STAGE_BYTES);
        if (p.npass == 2 && !(p.b_kmajor & 2)) {
          const bool ptr_ = (p.b_kmajor & 4) != 0;
#define PK(a, b) (ptr_ ? pack_bf16_trunc(a, b) : pack_bf16(a, b))
          // A' (K-major SW128 bf16, 128 rows x 64 virtual k): row r, virtual
          //   chunk 2g = bf16(hi) of real k 8g..8g+7, chunk 2g+1 = bf16(lo)
#pragma unroll
          for (int u = 0; u < (512 + XFORM_THREADS - 1) / XFORM_THREADS; ++u) {
            const int item = tid + u * XFORM_THREADS;
            if (item >= 512) break;
            const int r = item >> 2, g = item & 3, sw = r & 7;
            const uint32_t rowa = raw + r * 128;
            const uint4 x0 = lds128(rowa + (((2 * g) ^ sw) << 4));
            const uint4 x1 = lds128(rowa + (((2 * g + 1) ^ sw) << 4));
            const float f[8] = {__uint_as_float(x0.x), __uint_as_float(x0.y), __uint_as_float(x0.z),
                                __uint_as_float(x0.w), __uint_as_float(x1.x), __uint_as_float(x1.y),
                                __uint_as_float(x1.z), __uint_as_float(x1.w)};
            float h[8], l[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) {
              h[e] = trunc13(f[e]);
              l[e] = f[e] - h[e];
            }
            const uint32_t rowd = lo + r * 128;
            sts128(rowd + (((2 * g) ^ sw) << 4),
                   make_uint4(PK(h[0], h[1]), PK(h[2], h[3]), PK(h[4], h[5]),
                              PK(h[6], h[7])));
            sts128(rowd + (((2 * g + 1) ^ sw) << 4),
                   make_uint4(PK(l[0], l[1]), PK(l[2], l[3]), PK(l[4], l[5]),
                              PK(l[6], l[7])));
          }
          // B' (MN-major SW128 bf16, 64 virtual k x 128 n): virtual row
          //   16g+i = bf16(lo) of real k 8g+i, 16g+8+i = bf16(hi).  One item =
          //   8 consecutive n of one k: a 32-B granule of the raw tile (the
          //   BASE32B swizzle keeps granules whole) -> one 16-B chunk of B'.
#pragma unroll
          for (int u = 0; u < (512 + XFORM_THREADS - 1) / XFORM_THREADS; ++u) {
            const int item = tid + u * XFORM_THREADS;
            if (item >= 512) break;
            const int k = item >> 4, n0 = (item & 15) * 8;
            const int nn = n0 & 31;
            const uint32_t src = raw + A_BYTES + (n0 >> 5) * B_CHUNK_BYTES + k * 128 +
                                 (((nn >> 3) ^ (k & 3)) << 5);
            // lanes 4..7 of each 8-lane phase read the second 16 B first, so a
            // phase touches 8 distinct bank groups (no 2-way conflict)
            const uint32_t h1 = (threadIdx.x >> 2) & 1;
            const uint4 y0 = lds128(src + 16 * h1), y1 = lds128(src + 16 * (h1 ^ 1));
            const uint4 x0 = h1 ? y1 : y0, x1 = h1 ? y0 : y1;
            const float f[8] = {__uint_as_float(x0.x), __uint_as_float(x0.y), __uint_as_float(x0.z),
                                __uint_as_float(x0.w), __uint_as_float(x1.x), __uint_as_float(x1.y),
                                __uint_as_float(x1.z), __uint_as_float(x1.w)};
            float h[8], l[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) {
              h[e] = trunc13(f[e]);
              l[e] = f[e] - h[e];
            }
            const int vlo = 16 * (k >> 3) + (k & 7), vhi = vlo + 8;
            const int c = (n0 & 63) >> 3;
            const uint32_t base = lo + XA_BYTES + (n0 >> 6) * 8192;
            sts128(base + (vlo >> 3) * 1024 + (vlo & 7) * 128 + ((c ^ (vlo & 7)) << 4),
                   make_uint4(PK(l[0], l[1]), PK(l[2], l[3]), PK(l[4], l[5]),
                              PK(l[6], l[7])));
            sts128(base + (vhi >> 3) * 1024 + (vhi & 7) * 128 + ((c ^ (vhi & 7)) << 4),
                   make_uint4(PK(h[0], h[1]), PK(h[2], h[3]), PK(h[4], h[5]),
                              PK(h[6], h[7])));
          }
#undef PK
        } else if (p.npass == 3 && !(p.b_kmajor & 2)) {   // exp. 2: skip the split work
          constexpr int NV = (TMA_BYTES / 16 + XFORM_THREADS - 1) / XFORM_THREADS;
          uint4 x[NV];
#pragma unroll
          for (int u = 0; u < NV; ++u)
            if (tid + u * XFORM_THREADS < TMA_BYTES / 16) x[u] = lds128(raw + (tid + u * XFORM_THREADS) * 16);
#pragma unroll
          for (int u = 0; u < NV; ++u) {
            if (tid + u * XFORM_THREADS >= TMA_BYTES / 16) break;
            uint4 l;   // lo = x - trunc13(x): exact in fp32
            l.x = __float_as_uint(__uint_as_float(x[u].x) - __uint_as_float(x[u].x & 0xFFFFE000u));
            l.y = __float_as_uint(__uint_as_float(x[u].y) - __uint_as_float(x[u].y & 0xFFFFE000u));
            l.z = __float_as_uint(__uint_as_float(x[u].z) - __uint_as_float(x[u].z & 0xFFFFE000u));
            l.w = __float_as_uint(__uint_as_float(x[u].w) - __uint_as_float(x[u].w & 0xFFFFE000u));
            sts128(lo + (tid + u * XFORM_THREADS) * 16, l);
          }
        }
        fence_proxy_async_smem();   // generic st.shared -> visible to the tensor core
        named_bar(1, XFORM_THREADS);
        if (tid == 0) mbar_arrive_cluster(xform_leader0 + 8 * j);
      }
    }
    if (p.dbg && tid == 0) {
      float* d = p.dbg + 8 * cid + 4 + 2 * rank;
      d[0] = static_cast<float>(w_full);
      d[1] = static_cast<float>(w_lem);
    }
  } else {
    // ------------------------------------------------------ epilogue (own rows)
    const int q = warp & 3;
    const int row_in_tile = rank * BM_CTA + q * 32 + lane;
    const uint32_t tempty_leader0 = mapa(bar_tempty, 0);
    uint32_t chunk_it = 0;
    for (int t = cid; t < num_tiles; t += nclusters) {
      int mb, nb;
      tile_coords(t, p.tiles_m, p.tiles_n, p.band, mb, nb);
      const int row = mb * BM + row_in_tile;
      const bool row_ok = row < p.M;
      float* crow = p.C + static_cast<int64_t>(row) * p.ldc;
      for (int ch = 0; ch < nchunks; ++ch, ++chunk_it) {
        const uint32_t acc = chunk_it & 1, ause = chunk_it >> 1;
        mbar_wait(bar_tfull + 8 * acc, ause & 1);
        tc_fence_after();
        const bool add = (ch > 0) || p.accumulate;
#pragma unroll 1
        for (int c = 0; c < BN / 32; ++c) {
          uint32_t v[32];
          __syncwarp();
          tmem_ld32(tmem_base + (static_cast<uint32_t>(q * 32) << 16) + acc * BN + c * 32, v);
          const int col0 = nb * BN + c * 32;
          if (row_ok && col0 < p.N) {
            float* dst = crow + col0;
            if (p.vec_ok && col0 + 32 <= p.N) {
#pragma unroll
              for (int j = 0; j < 32; j += 4) {
                float4 o = make_float4(__uint_as_float(v[j]), __uint_as_float(v[j + 1]),
                                       __uint_as_float(v[j + 2]), __uint_as_float(v[j + 3]));
                if (add) {
                  const float4 c4 = *reinterpret_cast<const float4*>(dst + j);
                  o.x = c4.x + o.x;
                  o.y = c4.y + o.y;
                  o.z = c4.z + o.z;
                  o.w = c4.w + o.w;
                }
                *reinterpret_cast<float4*>(dst + j) = o;
              }
            } else {
              const int ncol = min(32, p.N - col0);
#pragma unroll
              for (int j = 0; j < 32; ++j) {
                if (j < ncol) {
                  float o = __uint_as_float(v[j]);
                  if (add) o = dst[j] + o;
                  dst[j] = o;
                }
              }
            }
          }
        }
        __syncwarp();
        tc_fence_before();
        mbar_arrive_cluster(tempty_leader0 + 8 * acc);
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  cluster_sync();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                 "n"(TMEM_COLS)
                 : "memory");
  }
}

}  // namespace sm2

void preload_sm2() {
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, sm2::leaf_gemm_2sm_kernel);
}

int launch_sm2(LaunchArgs& a) {
  using namespace sm2;
  int rc;
  CUtensorMap tmA, tmB;
  Params& p = a.p;
  // (2sm: b_kmajor is reused as an experiment bit field by tools/mma_prof.py)
  if ((rc = encode_2d(&tmA, a.A, p.K, p.M, a.lda, BK, BM_CTA))) return rc;
  if ((rc = encode_2d(&tmB, a.B, p.N, p.K, a.ldb, B_CHUNK, BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)))
    return rc;
  p.tiles_m = (p.M + BM - 1) / BM;
  p.tiles_n = (p.N + BN - 1) / BN;
  static std::atomic<int> configured[kMaxDevices];
  if (!configured[a.dev].load()) {
    cudaError_t e = cudaFuncSetAttribute(leaf_gemm_2sm_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return fail(NU_ECUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(e));
    configured[a.dev].store(1);
  }
  const int tiles = p.tiles_m * p.tiles_n;
  const int pairs = a.sms / 2;
  const int grid = 2 * (tiles < pairs ? tiles : pairs);
#if NU_LEAF2_PRESPLIT
  // experiment: one grow-only scratch per process, pre-pass on the same stream
  static char* scratch = nullptr;
  static size_t scratch_bytes = 0;
  const int K8 = (p.K + 7) / 8 * 8;
  const size_t need = 2ull * 2 * K8 * (static_cast<size_t>(p.M) + p.N) + 1024;
  if (need > scratch_bytes) {
    cudaStreamSynchronize(a.stream);
    if (scratch) cudaFree(scratch);
    if (cudaMalloc(&scratch, need) != cudaSuccess) return fail(NU_ENOMEM, "presplit scratch");
    scratch_bytes = need;
  }
  __nv_bfloat16* Ap = reinterpret_cast<__nv_bfloat16*>(scratch);
  __nv_bfloat16* Bp = Ap + static_cast<size_t>(p.M) * 2 * K8;
  presplit_a_kernel<<<1184, 256, 0, a.stream>>>(a.A, a.lda, p.M, p.K, K8, Ap);
  presplit_b_kernel<<<1184, 256, 0, a.stream>>>(a.B, a.ldb, p.K, p.N, K8, Bp);
  CUtensorMap tmAp, tmBp;
  if ((rc = encode_2d_bf16(&tmAp, Ap, 2 * K8, p.M, 2 * K8, 64, BM_CTA))) return rc;
  if ((rc = encode_2d_bf16(&tmBp, Bp, p.N, 2 * K8, p.N, 64, 2 * BK))) return rc;
  leaf_gemm_2sm_kernel<<<grid, NUM_THREADS, SMEM_BYTES, a.stream>>>(tmA, tmB, p, tmAp, tmBp);
#else
  leaf_gemm_2sm_kernel<<<grid, NUM_THREADS, SMEM_BYTES, a.stream>>>(tmA, tmB, p);
#endif
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : fail(NU_ECUDA, "leaf (2sm) launch: %s", cudaGetErrorString(e));
}

}  // namespace leaf
}  // namespace nu

// --------------------------------------------------------------------------
// Debug: raw tensor-core rate of the 2-CTA tf32 MMA (M=256, N=256, K=8) on
// fixed shared-memory operands, no pipeline — calibrates the 128-clk model.
namespace nu {
namespace leaf {
namespace sm2 {
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1)
    mma_rate_kernel(int n_mma, int mode, long long* out) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5;
  const uint32_t rank = cluster_ctarank();
  for (int i = threadIdx.x; i < 65536 / 4; i += blockDim.x) reinterpret_cast<float*>(smem)[i] = 0.f;
  if (threadIdx.x == 0) {
    mbar_init(smem_u32(&bar), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&slot)), "n"(256) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem = slot;
  if (rank == 0 && threadIdx.x == 0) {
    const uint32_t idesc = idesc_tf32(256, 256, 1u);
    const uint32_t a = smem_u32(smem), b = a + 16384, a2 = a + 32768, b2 = a + 49152;
    long long t0 = clock64();
    for (int i = 0; i < n_mma; ++i) {
      const uint64_t da = umma_desc((mode & 1) && (i % 3 == 2) ? a2 : a, 16, 1024);
      const uint64_t db = umma_desc((mode & 2) && (i % 3 == 0) ? b2 : b, B_CHUNK_BYTES, 512,
                                    LAYOUT_SW128_BASE32B);
      umma_tf32_2sm(tmem, da, db, idesc, i > 0);
    }
    umma_commit_pair(smem_u32(&bar));
    mbar_wait(smem_u32(&bar), 0);
    out[0] = clock64() - t0;
  } else if (rank == 1 && threadIdx.x == 0) {
    mbar_wait(smem_u32(&bar), 0);
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(256)
                 : "memory");
  }
}
}  // namespace sm2
}  // namespace leaf
}  // namespace nu

extern "C" int northup_debug_mma_rate(int n_mma, int mode, int grid, long long* out_dev) {
  cudaFuncSetAttribute(nu::leaf::sm2::mma_rate_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       70 * 1024);
  nu::leaf::sm2::mma_rate_kernel<<<grid, 128, 70 * 1024>>>(n_mma, mode, out_dev);
  cudaError_t e = cudaDeviceSynchronize();
  return e == cudaSuccess ? 0 : nu::fail(NU_ECUDA, "mma_rate: %s", cudaGetErrorString(e));
}
