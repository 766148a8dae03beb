// Leaf computation of the Northup tree on B200 (sm_100a).
//
// PAPER.md §IV-A: "at leafs, computation is executed on the
// GPU ... leverage the GPU's per-compute-unit local memory for each data
// block and manage the data movement explicitly".  On B200 the HBM -> SMEM
// edge is an explicit, descriptor-driven move (TMA), so the SMEM/TMEM leaf is
// a level of the tree: each CTA moves A (BM x BK) and B (BK x BN) tiles down
// into a shared-memory ring, splits them for 3xTF32, and accumulates
// C_tile += A_tile . B_tile in TMEM with tcgen05.mma kind::tf32.
//
// 3xTF32:   x = hi + lo,  hi = x with the low 13 mantissa bits
// cleared (exactly representable in TF32), lo = x - hi (exact in fp32), and
//     D += A_hi.B_hi + A_hi.B_lo + A_lo.B_hi
// The dropped A_lo.B_lo term and the TF32 rounding of lo are ~2^-20 of
// |a||b|, well inside the 1e-5 normwise bound of BASELINE.json.
//
// Partial-sum accumulation ("first computing partial results ... and
// then accumulate the partial sums"): the kernel accumulates in TMEM for
// exactly `kc` elements of K (one "chunk", aligned to the start of the call),
// then the epilogue warps add the chunk into C in fp32 round-to-nearest
// (C = acc for the first chunk unless `accumulate`).  Results are therefore
// bitwise identical for any plan whose K-panel boundaries are multiples of kc.
//
// Warp roles (one CTA per SM, persistent over output tiles):
//   warp 0      TMA producer (one elected lane)
//   warp 1      TMEM allocator + MMA issuer (one elected lane)
//   warps 2-5   transform: in-place hi, lo into a second buffer
//   warps 6-9   epilogue: TMEM -> registers -> C (global), fp32 RN add
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "leaf_common.cuh"
#include "northup_internal.h"

namespace nu {
namespace leaf {
namespace sm1 {

constexpr int BM = 128;              // UMMA M (cta_group::1)
constexpr int BN = 256;              // UMMA N
constexpr int STAGES = 2;
constexpr int A_BYTES = BM * BK * 4;               // 16 KiB
constexpr int B_BYTES = BN * BK * 4;               // 32 KiB
constexpr int TMA_BYTES = A_BYTES + B_BYTES;       // bytes landed per stage
constexpr int STAGE_BYTES = 2 * TMA_BYTES;         // raw (hi in place) + lo
constexpr int NUM_THREADS = 320;
constexpr int XFORM_THREADS = 128;
constexpr int EPI_THREADS = 128;
constexpr int TMEM_COLS = 512;                     // 2 accumulators x BN fp32 columns
constexpr int BAR_BYTES = 1024;
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + BAR_BYTES + 1024;  // + 1 KiB alignment slack

static_assert(BK == 32, "A tile rows are one 128-B swizzle atom wide");
static_assert(SMEM_BYTES <= 227 * 1024, "shared memory budget");


// ------------------------------------------------------------------- kernel
__global__ void __launch_bounds__(NUM_THREADS, 1)
    leaf_gemm_1sm_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                     const Params p) {
  extern __shared__ uint8_t smem_raw[];
  // 1024-byte alignment for the 128-B swizzle atoms.
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  uint8_t* bars = smem + STAGES * STAGE_BYTES;
  const uint32_t bar_full = smem_u32(bars);            // [STAGES] TMA landed
  const uint32_t bar_xform = bar_full + 8 * STAGES;    // [STAGES] split done
  const uint32_t bar_empty = bar_xform + 8 * STAGES;   // [STAGES] MMAs done reading
  const uint32_t bar_tfull = bar_empty + 8 * STAGES;   // [2] accumulator ready
  const uint32_t bar_tempty = bar_tfull + 16;          // [2] accumulator drained
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 8 * (3 * STAGES + 4));

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(bar_full + 8 * s, 1);
      mbar_init(bar_xform + 8 * s, XFORM_THREADS);
      mbar_init(bar_empty + 8 * s, 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(bar_tfull + 8 * a, 1);
      mbar_init(bar_tempty + 8 * a, EPI_THREADS);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "n"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  const int num_tiles = p.tiles_m * p.tiles_n;
  const int nkb = (p.K + BK - 1) / BK;
  const int nchunks = (nkb + p.kb_per_chunk - 1) / p.kb_per_chunk;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      uint32_t it = 0;
      for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
        int mb, nb;
        tile_coords(t, p.tiles_m, p.tiles_n, p.band, mb, nb);
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const uint32_t s = it % STAGES, use = it / STAGES;
          mbar_wait(bar_empty + 8 * s, (use & 1) ^ 1);
          const uint32_t full = bar_full + 8 * s;
          mbar_arrive_expect_tx(full, TMA_BYTES);
          const uint32_t sa = smem_u32(smem + s * STAGE_BYTES);
          const uint32_t sb = sa + A_BYTES;
          tma_load_2d(sa, &tmA, full, kb * BK, mb * BM);
          if (p.b_kmajor) {
            tma_load_2d(sb, &tmB, full, kb * BK, nb * BN);
          } else {
#pragma unroll
            for (int c = 0; c < BN / B_CHUNK; ++c)
              tma_load_2d(sb + c * B_CHUNK_BYTES, &tmB, full, nb * BN + c * B_CHUNK, kb * BK);
          }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------- MMA issuer
    if (lane == 0) {
      const uint32_t idesc = idesc_tf32(BM, BN, p.b_kmajor ? 0u : 1u);
      uint32_t it = 0, chunk_it = 0;
      for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
        for (int ch = 0; ch < nchunks; ++ch, ++chunk_it) {
          const uint32_t acc = chunk_it & 1, ause = chunk_it >> 1;
          mbar_wait(bar_tempty + 8 * acc, (ause & 1) ^ 1);
          tc_fence_after();
          const uint32_t tmem_d = tmem_base + acc * BN;
          const int kb0 = ch * p.kb_per_chunk;
          const int kb1 = min(nkb, kb0 + p.kb_per_chunk);
          for (int kb = kb0; kb < kb1; ++kb, ++it) {
            const uint32_t s = it % STAGES, use = it / STAGES;
            mbar_wait(bar_xform + 8 * s, use & 1);
            tc_fence_after();
            const uint32_t a_hi = smem_u32(smem + s * STAGE_BYTES);
            const uint32_t b_hi = a_hi + A_BYTES;
            const uint32_t a_lo = a_hi + TMA_BYTES;
            const uint32_t b_lo = b_hi + TMA_BYTES;
#pragma unroll
            for (int k = 0; k < BK / UMMA_K; ++k) {
              // A: K-major SW128, advance 32 B per k-step inside the atom row.
              // B: MN-major SW128_BASE32B, LBO = stride between 32-column
              //    chunks, SBO = stride between 4-row atoms (512 B); a k-step
              //    (8 rows) advances 1024 B.
              const uint64_t dah = umma_desc(a_hi + k * 32, 16, 1024);
              const uint64_t dal = umma_desc(a_lo + k * 32, 16, 1024);
              const uint64_t dbh = p.b_kmajor ? umma_desc(b_hi + k * 32, 16, 1024)
                                              : umma_desc(b_hi + k * 1024, B_CHUNK_BYTES, 512,
                                                          LAYOUT_SW128_BASE32B);
              const uint64_t dbl = p.b_kmajor ? umma_desc(b_lo + k * 32, 16, 1024)
                                              : umma_desc(b_lo + k * 1024, B_CHUNK_BYTES, 512,
                                                          LAYOUT_SW128_BASE32B);
              const uint32_t first = (kb == kb0 && k == 0) ? 0u : 1u;
              if (p.npass == 3) {
                umma_tf32(tmem_d, dal, dbh, idesc, first);   // small terms first
                umma_tf32(tmem_d, dah, dbl, idesc, 1u);
                umma_tf32(tmem_d, dah, dbh, idesc, 1u);
              } else {
                umma_tf32(tmem_d, dah, dbh, idesc, first);
              }
            }
            umma_commit(bar_empty + 8 * s);   // frees the stage when these MMAs retire
          }
          umma_commit(bar_tfull + 8 * acc);   // chunk accumulated -> epilogue
        }
      }
    }
  } else if (warp < 6) {
    // --------------------------------------------------------------- transform
    const int tid = threadIdx.x - 64;
    uint32_t it = 0;
    for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
      for (int kb = 0; kb < nkb; ++kb, ++it) {
        const uint32_t s = it % STAGES, use = it / STAGES;
        mbar_wait(bar_full + 8 * s, use & 1);
        uint4* raw = reinterpret_cast<uint4*>(smem + s * STAGE_BYTES);
        uint4* lo = reinterpret_cast<uint4*>(smem + s * STAGE_BYTES + TMA_BYTES);
        if (p.npass == 3) {
#pragma unroll 4
          for (int i = tid; i < TMA_BYTES / 16; i += XFORM_THREADS) {
            uint4 x = raw[i];
            uint4 h, l;
            h.x = x.x & 0xFFFFE000u;
            h.y = x.y & 0xFFFFE000u;
            h.z = x.z & 0xFFFFE000u;
            h.w = x.w & 0xFFFFE000u;
            l.x = __float_as_uint(__uint_as_float(x.x) - __uint_as_float(h.x));
            l.y = __float_as_uint(__uint_as_float(x.y) - __uint_as_float(h.y));
            l.z = __float_as_uint(__uint_as_float(x.z) - __uint_as_float(h.z));
            l.w = __float_as_uint(__uint_as_float(x.w) - __uint_as_float(h.w));
            raw[i] = h;
            lo[i] = l;
          }
        }
        if (p.dbg && blockIdx.x == 0 && it == 0) {
          __syncwarp();
          asm volatile("bar.sync 1, 128;" ::: "memory");
          const float* src = reinterpret_cast<const float*>(smem + s * STAGE_BYTES);
          for (int i = tid; i < STAGE_BYTES / 4; i += XFORM_THREADS) p.dbg[i] = src[i];
        }
        fence_proxy_async_smem();   // generic-proxy writes -> visible to tcgen05 reads
        mbar_arrive(bar_xform + 8 * s);
      }
    }
  } else {
    // ---------------------------------------------------------------- epilogue
    const int q = warp & 3;          // TMEM lane quarter this warp may access
    const int row_in_tile = q * 32 + lane;
    uint32_t chunk_it = 0;
    for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
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
          __syncwarp();   // tcgen05.ld is .sync.aligned: the warp must be converged
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
        mbar_arrive(bar_tempty + 8 * acc);
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                 "n"(TMEM_COLS)
                 : "memory");
  }
}

}  // namespace sm1

void preload_sm1() {
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, sm1::leaf_gemm_1sm_kernel);
}

int launch_sm1(LaunchArgs& a) {
  using namespace sm1;
  int rc;
  CUtensorMap tmA, tmB;
  Params& p = a.p;
  if ((rc = encode_2d(&tmA, a.A, p.K, p.M, a.lda, BK, BM))) return rc;
  if (p.b_kmajor) {
    if ((rc = encode_2d(&tmB, a.B, p.K, p.N, a.ldb, BK, BN))) return rc;
  } else {
    if ((rc = encode_2d(&tmB, a.B, p.N, p.K, a.ldb, B_CHUNK, BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)))
      return rc;
  }
  p.tiles_m = (p.M + BM - 1) / BM;
  p.tiles_n = (p.N + BN - 1) / BN;
  static std::atomic<int> configured[kMaxDevices];
  if (!configured[a.dev].load()) {
    cudaError_t e = cudaFuncSetAttribute(leaf_gemm_1sm_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return fail(NU_ECUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(e));
    configured[a.dev].store(1);
  }
  const int tiles = p.tiles_m * p.tiles_n;
  const int grid = tiles < a.sms ? tiles : a.sms;
  leaf_gemm_1sm_kernel<<<grid, NUM_THREADS, SMEM_BYTES, a.stream>>>(tmA, tmB, p);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : fail(NU_ECUDA, "leaf (1sm) launch: %s", cudaGetErrorString(e));
}

}  // namespace leaf
}  // namespace nu
