// Leaf kernel v2: the CTA-pair kernel of leaf_2sm.cu (v1) with the raw tiles
// loaded by the split warps themselves instead of TMA.
//
// Profiling v1 (profiles/r01_leaf_cycles.txt) showed the split to be the
// bottleneck and shared memory bandwidth to be the reason: per 32-K stage a
// CTA's shared memory carried TMA writes 32 KiB + split reads 32 KiB + split
// writes 32 KiB + MMA reads 64 KiB.  Here the split warps load the stage from
// global memory (L2) straight into registers, write the raw tiles (the tf32
// hi.hi operands, in the same swizzled layouts TMA produced) and the bf16
// cross-term tiles, so shared memory carries 64 + 64 KiB per stage — the
// tensor-core floor (1024 clk per stage) instead of 1250.  Warp 0 keeps the
// tensor maps only to prefetch future stages into L2
// (cp.async.bulk.prefetch.tensor), hiding DRAM latency from the loads.
//
// Same arithmetic as v1 with npass = 2 (R19/R21), same epilogue,
// same chunked accumulation: results are bitwise identical to v1.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "leaf_2sm_common.cuh"
#include "leaf_common.cuh"
#include "northup_internal.h"

namespace nu {
namespace leaf {
namespace sm3 {

using namespace sm2;

constexpr int BM = 256, BN = 256, BM_CTA = 128, BN_CTA = 128;
#ifndef NU_LEAF3_STAGES
#define NU_LEAF3_STAGES 3
#endif
constexpr int STAGES = NU_LEAF3_STAGES;
constexpr int A_BYTES = BM_CTA * BK * 4;           // raw A 16 KiB (K-major SW128)
constexpr int B_BYTES = BN_CTA * BK * 4;           // raw B 16 KiB (MN-major SW128_32B chunks)
constexpr int XA_BYTES = BM_CTA * 2 * BK * 2;      // A' bf16 16 KiB
constexpr int XB_BYTES = 2 * BK * BN_CTA * 2;      // B' bf16 16 KiB
constexpr int STAGE_BYTES = A_BYTES + B_BYTES + XA_BYTES + XB_BYTES;   // 64 KiB
#ifndef NU_LEAF3_SPLIT_WARPS
#define NU_LEAF3_SPLIT_WARPS 8
#endif
constexpr int SPLIT_WARPS = NU_LEAF3_SPLIT_WARPS;
constexpr int SPLIT_THREADS = 32 * SPLIT_WARPS;
constexpr int EPI_WARP0 = 2 + SPLIT_WARPS;
constexpr int EPI_THREADS = 128;
constexpr int NUM_THREADS = 32 * (EPI_WARP0 + 4);
constexpr int A_ITEMS = BM_CTA * BK / 4;           // (row, 4 k) items: 1024
constexpr int B_ITEMS = BK * BN_CTA / 4;           // (k, 4 n) items: 1024
constexpr int AI = A_ITEMS / SPLIT_THREADS;        // per thread
constexpr int BI = B_ITEMS / SPLIT_THREADS;
#ifndef NU_LEAF3_PF
#define NU_LEAF3_PF 3
#endif
constexpr int PF = NU_LEAF3_PF;                    // L2 prefetch distance (stages), 0 = off
constexpr int TMEM_COLS = 512;
constexpr int BAR_BYTES = 256;
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + BAR_BYTES + 1024;
static_assert(SMEM_BYTES <= 227 * 1024, "shared memory budget");
static_assert(A_ITEMS % SPLIT_THREADS == 0 && B_ITEMS % SPLIT_THREADS == 0, "item split");

__device__ __forceinline__ float4 ldg_f4(const float* p) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p));
  return v;
}

__device__ __forceinline__ void prefetch_l2_2d(const CUtensorMap* map, int c0, int c1) {
  asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global [%0, {%1, %2}];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(c0), "r"(c1)
               : "memory");
}

// Registers of one stage for one split thread: AI items of 4 consecutive k
// of one A row and BI items of 4 consecutive n of one B row.  A warp's 32
// items are 512 contiguous bytes of A (4 rows) or of B (one k-row): every
// load is fully coalesced and every shared-memory store below is free of
// bank conflicts (8-lane phases cover 8 distinct 16-B slots).
struct StageRegs {
  float a[AI][4];
  float b[BI][4];
};

// Issue the loads of the thread's part of stage (row0, col0, k0).  Nothing
// here reads the loaded registers, so the loads stay in flight until
// store_stage (which also zeroes elements past K / N inside a vector).
__device__ __forceinline__ void load_stage(const Params& p, int tid, int row0, int col0, int k0,
                                           StageRegs& r) {
#pragma unroll
  for (int u = 0; u < AI; ++u) {
    const int item = tid + u * SPLIT_THREADS;
    const int row = row0 + (item >> 3), k = k0 + 4 * (item & 7);
    float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
    if (row < p.M && k < p.K) x = ldg_f4(p.A + static_cast<int64_t>(row) * p.lda + k);
    r.a[u][0] = x.x; r.a[u][1] = x.y; r.a[u][2] = x.z; r.a[u][3] = x.w;
  }
#pragma unroll
  for (int u = 0; u < BI; ++u) {
    const int item = tid + u * SPLIT_THREADS;
    const int k = k0 + (item >> 5), n = col0 + 4 * (item & 31);
    float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
    if (k < p.K && n < p.N) x = ldg_f4(p.B + static_cast<int64_t>(k) * p.ldb + n);
    r.b[u][0] = x.x; r.b[u][1] = x.y; r.b[u][2] = x.z; r.b[u][3] = x.w;
  }
}

__device__ __forceinline__ uint4 as_u4(const float* f) {
  return make_uint4(__float_as_uint(f[0]), __float_as_uint(f[1]), __float_as_uint(f[2]),
                    __float_as_uint(f[3]));
}

// Write one stage: raw A (K-major SW128), raw B (MN-major SW128_32B chunks),
// A' and B' (bf16, the R21 layouts of v1).
__device__ __forceinline__ void store_stage(uint32_t st, int tid, const StageRegs& r, int kmax,
                                            int nmax) {
  // kmax / nmax: valid k / n extents of this stage (elements beyond are zero,
  // the TMA OOB fill of v1)
  const uint32_t rawA = st, rawB = st + A_BYTES, xa = st + A_BYTES + B_BYTES, xb = xa + XA_BYTES;
#pragma unroll
  for (int u = 0; u < AI; ++u) {
    const int item = tid + u * SPLIT_THREADS;
    const int row = item >> 3, c = item & 7, sw = row & 7, g = c >> 1, half = c & 1;
    float f[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) f[e] = (4 * c + e < kmax) ? r.a[u][e] : 0.f;
    float h[4], l[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      h[e] = trunc13(f[e]);
      l[e] = f[e] - h[e];
    }
    sts128(rawA + row * 128 + ((c ^ sw) << 4), as_u4(f));
    sts64(xa + row * 128 + (((2 * g) ^ sw) << 4) + half * 8, pack_bf16(h[0], h[1]), pack_bf16(h[2], h[3]));
    sts64(xa + row * 128 + (((2 * g + 1) ^ sw) << 4) + half * 8, pack_bf16(l[0], l[1]),
          pack_bf16(l[2], l[3]));
  }
#pragma unroll
  for (int u = 0; u < BI; ++u) {
    const int item = tid + u * SPLIT_THREADS;
    const int k = item >> 5, n0 = 4 * (item & 31), nn = n0 & 31;
    float f[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) f[e] = (n0 + e < nmax) ? r.b[u][e] : 0.f;
    float h[4], l[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      h[e] = trunc13(f[e]);
      l[e] = f[e] - h[e];
    }
    sts128(rawB + (n0 >> 5) * B_CHUNK_BYTES + k * 128 + ((((nn >> 3) ^ (k & 3)) << 5) | ((nn & 4) << 2)),
           as_u4(f));
    const int vlo = 16 * (k >> 3) + (k & 7), vhi = vlo + 8;
    const int c = (n0 & 63) >> 3;
    const uint32_t base = xb + (n0 >> 6) * 8192 + ((n0 >> 2) & 1) * 8;
    sts64(base + (vlo >> 3) * 1024 + (vlo & 7) * 128 + ((c ^ (vlo & 7)) << 4), pack_bf16(l[0], l[1]),
          pack_bf16(l[2], l[3]));
    sts64(base + (vhi >> 3) * 1024 + (vhi & 7) * 128 + ((c ^ (vhi & 7)) << 4), pack_bf16(h[0], h[1]),
          pack_bf16(h[2], h[3]));
  }
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(NUM_THREADS, 1)
    leaf_gemm_2sm_ldg_kernel(const __grid_constant__ CUtensorMap tmA,
                             const __grid_constant__ CUtensorMap tmB, const Params p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  uint8_t* bars = smem + STAGES * STAGE_BYTES;
  const uint32_t bar_empty = smem_u32(bars);          // [STAGES] each CTA: leader's commit
  const uint32_t bar_ready = bar_empty + 8 * STAGES;  // [STAGES] leader: both CTAs wrote the stage
  const uint32_t bar_tfull = bar_ready + 8 * STAGES;  // [2] each CTA
  const uint32_t bar_tempty = bar_tfull + 16;         // [2] leader
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 8 * (2 * STAGES + 4));

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;

  if (threadIdx.x == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(bar_empty + 8 * s, 1);
      mbar_init(bar_ready + 8 * s, 2);
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
    // ------------------------------------ L2 prefetcher (paced by the ring)
    if (lane == 0) {
      uint32_t it = 0;
      int pt = cid, pkb = 0;   // the stage to prefetch: PF ahead of `it`
      for (int i = 0; i < PF && pt < num_tiles; ++i) {
        if (++pkb == nkb) { pkb = 0; pt += nclusters; }
      }
      for (int t = cid; t < num_tiles; t += nclusters) {
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const uint32_t s = it % STAGES, use = it / STAGES;
          mbar_wait(bar_empty + 8 * s, (use & 1) ^ 1);
          if (PF > 0 && pt < num_tiles) {
            int mb, nb;
            tile_coords(pt, p.tiles_m, p.tiles_n, p.band, mb, nb);
            prefetch_l2_2d(&tmA, pkb * BK, mb * BM + rank * BM_CTA);
#pragma unroll
            for (int c = 0; c < BN_CTA / B_CHUNK; ++c)
              prefetch_l2_2d(&tmB, nb * BN + rank * BN_CTA + c * B_CHUNK, pkb * BK);
            if (++pkb == nkb) { pkb = 0; pt += nclusters; }
          }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------- MMA issuer (leader CTA only)
    if (leader && lane == 0) {
      const uint32_t idesc = idesc_tf32(BM, BN, 1u);
      const uint32_t idesc_bf = idesc_bf16(BM, BN);
      uint32_t it = 0, chunk_it = 0;
      long long w_rd = 0, w_te = 0, t_beg = clock64();
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
            const uint32_t s = it % STAGES, use = it / STAGES;
            c0 = clock64();
            mbar_wait_cluster(bar_ready + 8 * s, use & 1);
            w_rd += clock64() - c0;
            tc_fence_after();
            const uint32_t st = smem_u32(smem + s * STAGE_BYTES);
            const uint32_t a_raw = st, b_raw = st + A_BYTES, xa = st + A_BYTES + B_BYTES,
                           xb = xa + XA_BYTES;
            // same MMA order as v1 (all hi.hi of the stage, then the cross
            // terms), so v1 and v2 round identically
#pragma unroll
            for (int k = 0; k < BK / UMMA_K; ++k)
              umma_tf32_2sm(tmem_d, umma_desc(a_raw + k * 32, 16, 1024),
                            umma_desc(b_raw + k * 1024, B_CHUNK_BYTES, 512, LAYOUT_SW128_BASE32B),
                            idesc, (kb == kb0 && k == 0) ? 0u : 1u);
#pragma unroll
            for (int k = 0; k < BK / UMMA_K; ++k)
              umma_bf16_2sm(tmem_d, umma_desc(xa + k * 32, 16, 1024),
                            umma_desc(xb + k * 2048, 8192, 1024), idesc_bf, 1u);
            umma_commit_pair(bar_empty + 8 * s);
          }
          umma_commit_pair(bar_tfull + 8 * acc);
        }
      }
      if (p.dbg) {
        float* d = p.dbg + 8 * cid;
        d[0] = static_cast<float>(clock64() - t_beg);
        d[1] = static_cast<float>(w_rd);
        d[2] = static_cast<float>(w_te);
        d[3] = static_cast<float>(it);
      }
    }
  } else if (warp < EPI_WARP0) {
    // -------------------------------- split: global -> registers -> 4 tiles
    // Three register sets rotate so the loads of stage i+2 are in flight
    // while stage i is written (the L2 prefetcher runs further ahead).
    const int tid = threadIdx.x - 64;
    const uint32_t ready_leader0 = mapa(bar_ready, 0);
    long long w_em = 0, w_all = clock64();
    const int my_tiles = cid < num_tiles ? (num_tiles - cid + nclusters - 1) / nclusters : 0;
    const int total = my_tiles * nkb;
    auto load_it = [&](int i, StageRegs& r) {
      if (i >= total) return;
      const int t = cid + (i / nkb) * nclusters, kb = i % nkb;
      int mb, nb;
      tile_coords(t, p.tiles_m, p.tiles_n, p.band, mb, nb);
      load_stage(p, tid, mb * BM + rank * BM_CTA, nb * BN + rank * BN_CTA, kb * BK, r);
    };
    auto store_it = [&](int i, const StageRegs& r) {
      const uint32_t s = i % STAGES, use = i / STAGES;
      const int t = cid + (i / nkb) * nclusters, kb = i % nkb;
      int mb, nb;
      tile_coords(t, p.tiles_m, p.tiles_n, p.band, mb, nb);
      const int kmax = p.K - kb * BK, nmax = p.N - (nb * BN + rank * BN_CTA);
      long long c0 = clock64();
      mbar_wait(bar_empty + 8 * s, (use & 1) ^ 1);
      w_em += clock64() - c0;
      store_stage(smem_u32(smem + s * STAGE_BYTES), tid, r, kmax, nmax);
      fence_proxy_async_smem();   // generic st.shared -> visible to the tensor core
      named_bar(1, SPLIT_THREADS);
      if (tid == 0) mbar_arrive_cluster(ready_leader0 + 8 * s);
    };
    StageRegs r0, r1, r2;
    load_it(0, r0);
    load_it(1, r1);
    for (int i = 0; i < total; i += 3) {
      load_it(i + 2, r2);
      store_it(i, r0);
      if (i + 1 >= total) break;
      load_it(i + 3, r0);
      store_it(i + 1, r1);
      if (i + 2 >= total) break;
      load_it(i + 4, r1);
      store_it(i + 2, r2);
    }
    if (p.dbg && tid == 0) {
      float* d = p.dbg + 8 * cid + 4 + 2 * rank;
      d[0] = static_cast<float>(clock64() - w_all);
      d[1] = static_cast<float>(w_em);
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

}  // namespace sm3

void preload_sm3() {
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, sm3::leaf_gemm_2sm_ldg_kernel);
}

int launch_sm3(LaunchArgs& a) {
  using namespace sm3;
  int rc;
  CUtensorMap tmA, tmB;
  Params& p = a.p;
  // tensor maps only feed the L2 prefetcher
  if ((rc = encode_2d(&tmA, a.A, p.K, p.M, a.lda, BK, BM_CTA))) return rc;
  if ((rc = encode_2d(&tmB, a.B, p.N, p.K, a.ldb, B_CHUNK, BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)))
    return rc;
  p.tiles_m = (p.M + BM - 1) / BM;
  p.tiles_n = (p.N + BN - 1) / BN;
  static std::atomic<int> configured[kMaxDevices];
  if (!configured[a.dev].load()) {
    cudaError_t e = cudaFuncSetAttribute(leaf_gemm_2sm_ldg_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return fail(NU_ECUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(e));
    configured[a.dev].store(1);
  }
  const int tiles = p.tiles_m * p.tiles_n;
  const int pairs = a.sms / 2;
  const int grid = 2 * (tiles < pairs ? tiles : pairs);
  leaf_gemm_2sm_ldg_kernel<<<grid, NUM_THREADS, SMEM_BYTES, a.stream>>>(tmA, tmB, p);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : fail(NU_ECUDA, "leaf (2sm ldg) launch: %s", cudaGetErrorString(e));
}

}  // namespace leaf
}  // namespace nu
