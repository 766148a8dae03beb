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

#include "northup_internal.h"

namespace nu {
namespace leaf {

constexpr int BM = 128;              // UMMA M (cta_group::1)
constexpr int BN = 256;              // UMMA N
constexpr int BK = 32;               // K elements per pipeline stage (128 B rows)
constexpr int UMMA_K = 8;            // K per tcgen05.mma kind::tf32
constexpr int STAGES = 2;
constexpr int A_BYTES = BM * BK * 4;               // 16 KiB
constexpr int B_BYTES = BN * BK * 4;               // 32 KiB
constexpr int TMA_BYTES = A_BYTES + B_BYTES;       // bytes landed per stage
constexpr int STAGE_BYTES = 2 * TMA_BYTES;         // raw (hi in place) + lo
constexpr int B_CHUNK = 32;                        // N columns per 128-B swizzle atom
constexpr int B_CHUNK_BYTES = B_CHUNK * BK * 4;    // 4 KiB: one TMA box of B
constexpr int NUM_THREADS = 320;
constexpr int XFORM_THREADS = 128;
constexpr int EPI_THREADS = 128;
constexpr int TMEM_COLS = 512;                     // 2 accumulators x BN fp32 columns
constexpr int BAR_BYTES = 1024;
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + BAR_BYTES + 1024;  // + 1 KiB alignment slack
constexpr int RASTER_BAND = 4;                     // n-blocks per raster band (L2 reuse)

static_assert(BK == 32, "A tile rows are one 128-B swizzle atom wide");
static_assert(SMEM_BYTES <= 227 * 1024, "shared memory budget");

struct Params {
  float* C;
  int64_t ldc;
  int M, N, K;
  int kb_per_chunk;   // k-blocks (of BK) per TMEM accumulation chunk
  int accumulate;     // 1: C += A.B ; 0: C = A.B
  int tiles_m, tiles_n;
  int vec_ok;         // C base and ldc allow 16-byte vector access
  int npass;          // 3 = 3xTF32 (product path), 1 = plain TF32 (negative test)
  int b_kmajor;       // debug: B given as N x K (K-major) instead of K x N
  float* dbg;         // debug: dump of stage 0 after the split (NULL in production)
};

// ---------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Wait for the phase with the given parity to complete.  A watchdog traps
// after ~4 s instead of hanging the GPU if a pipeline invariant is broken.
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done = 0;
  uint64_t t0 = 0;
  for (uint32_t it = 0;; ++it) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
    if (done) return;
    if ((it & 1023u) == 0) {
      const uint64_t t = globaltimer();
      if (it == 0) t0 = t;
      else if (t - t0 > 4000000000ull) __trap();
    }
  }
}

__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, uint32_t bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}

__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// UMMA shared-memory matrix descriptor (sm_100): start>>4 [0,14), LBO>>4
// [16,30), SBO>>4 [32,46), version=1 [46,48), layout [61,64):
//   2 = SWIZZLE_128B (K-major A: 16-B granules XOR row%8),
//   1 = SWIZZLE_128B_BASE32B (MN-major 32-bit B: 32-B granules XOR row%4 —
//       the only MN-major smem layout the tensor core accepts for tf32).
constexpr uint32_t LAYOUT_SW128 = 2;
constexpr uint32_t LAYOUT_SW128_BASE32B = 1;
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo,
                                              uint32_t layout = LAYOUT_SW128) {
  uint64_t d = 0;
  d |= static_cast<uint64_t>((saddr >> 4) & 0x3FFFu);
  d |= static_cast<uint64_t>((lbo >> 4) & 0x3FFFu) << 16;
  d |= static_cast<uint64_t>((sbo >> 4) & 0x3FFFu) << 32;
  d |= static_cast<uint64_t>(1) << 46;
  d |= static_cast<uint64_t>(layout) << 61;
  return d;
}

// Instruction descriptor, kind::tf32: D f32 [4,6)=1, A tf32 [7,10)=2,
// B tf32 [10,13)=2, A K-major [15]=0, B MN-major [16]=1, N>>3 [17,23), M>>4 [24,29).
__host__ __device__ constexpr uint32_t idesc_tf32(int m, int n, uint32_t b_mn_major = 1) {
  return (1u << 4) | (2u << 7) | (2u << 10) | (0u << 15) | (b_mn_major << 16) |
         (static_cast<uint32_t>(n >> 3) << 17) | (static_cast<uint32_t>(m >> 4) << 24);
}

__device__ __forceinline__ void umma_tf32(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc,
                                          uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(da), "l"(db), "r"(idesc), "r"(accum)
      : "memory");
}

__device__ __forceinline__ void umma_commit(uint32_t bar) {
  asm volatile(
      "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar)
      : "memory");
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
      "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
        "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
        "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ void tile_coords(int t, int tiles_m, int tiles_n, int& mb, int& nb) {
  const int band = t / (tiles_m * RASTER_BAND);
  const int rem = t - band * tiles_m * RASTER_BAND;
  const int n0 = band * RASTER_BAND;
  const int bw = min(RASTER_BAND, tiles_n - n0);
  mb = rem / bw;
  nb = n0 + rem % bw;
}

// ------------------------------------------------------------------- kernel
__global__ void __launch_bounds__(NUM_THREADS, 1)
    leaf_gemm_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
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
        tile_coords(t, p.tiles_m, p.tiles_n, mb, nb);
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
      tile_coords(t, p.tiles_m, p.tiles_n, mb, nb);
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

}  // namespace leaf

// --------------------------------------------------------------- host side
static PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

static int get_encode() {
  if (g_encode) return 0;
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaError_t e = cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fn, 12000,
                                                   cudaEnableDefault, &q);
  if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn) {
    set_error("cuTensorMapEncodeTiled unavailable: %s", cudaGetErrorString(e));
    return NU_ECUDA;
  }
  g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  return 0;
}

static int encode_2d(CUtensorMap* map, const float* base, uint64_t inner, uint64_t outer,
                     uint64_t ld_elems, uint32_t box_inner, uint32_t box_outer,
                     CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {ld_elems * 4};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = g_encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims,
                        strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d): base=%p inner=%llu outer=%llu ld=%llu", (int)r,
              (const void*)base, (unsigned long long)inner, (unsigned long long)outer,
              (unsigned long long)ld_elems);
    return NU_EINVAL;
  }
  return 0;
}

bool leaf_tma_legal(const void* p, int64_t ld) {
  return (reinterpret_cast<uintptr_t>(p) % 16 == 0) && (ld % 4 == 0) && ld > 0;
}

int leaf_gemm_launch_dbg(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                         int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t kc,
                         int npass, int b_kmajor, float* dbg, cudaStream_t stream);

int leaf_gemm_launch(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                     int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t kc,
                     int npass, cudaStream_t stream) {
  return leaf_gemm_launch_dbg(A, lda, B, ldb, C, ldc, M, N, K, accumulate, kc, npass, 0, nullptr,
                              stream);
}

int leaf_gemm_launch_dbg(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                         int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t kc,
                         int npass, int b_kmajor, float* dbg, cudaStream_t stream) {
  using namespace leaf;
  if (M < 0 || N < 0 || K < 0) return set_error("negative dimension"), NU_EINVAL;
  if (M == 0 || N == 0) return 0;
  if (K == 0) {
    if (accumulate) return 0;
    cudaError_t e = cudaMemset2DAsync(C, ldc * 4, 0, N * 4, M, stream);
    return e == cudaSuccess ? 0 : (set_error("memset: %s", cudaGetErrorString(e)), NU_ECUDA);
  }
  if (M > INT32_MAX || N > INT32_MAX || K > INT32_MAX)
    return set_error("dimension exceeds int32 TMA coordinates"), NU_EINVAL;
  if (!leaf_tma_legal(A, lda) || !leaf_tma_legal(B, ldb))
    return set_error("leaf operands need 16-B aligned base and ld %% 4 == 0"), NU_EINVAL;
  if (lda < K || ldb < (b_kmajor ? K : N) || ldc < N)
    return set_error("leading dimension too small"), NU_EINVAL;
  int rc = get_encode();
  if (rc) return rc;
  CUtensorMap tmA, tmB;
  if ((rc = encode_2d(&tmA, A, K, M, lda, BK, BM))) return rc;
  if (b_kmajor) {
    if ((rc = encode_2d(&tmB, B, K, N, ldb, BK, BN))) return rc;
  } else {
    if ((rc = encode_2d(&tmB, B, N, K, ldb, B_CHUNK, BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)))
      return rc;
  }

  if (kc <= 0) kc = K;
  int64_t kbpc = (kc + BK - 1) / BK;
  if (kbpc < 1) kbpc = 1;
  if (kbpc > INT32_MAX) kbpc = INT32_MAX;

  Params p;
  p.C = C;
  p.ldc = ldc;
  p.M = static_cast<int>(M);
  p.N = static_cast<int>(N);
  p.K = static_cast<int>(K);
  p.kb_per_chunk = static_cast<int>(kbpc);
  p.accumulate = accumulate ? 1 : 0;
  p.tiles_m = static_cast<int>((M + BM - 1) / BM);
  p.tiles_n = static_cast<int>((N + BN - 1) / BN);
  p.vec_ok = (reinterpret_cast<uintptr_t>(C) % 16 == 0) && (ldc % 4 == 0);
  p.npass = npass == 1 ? 1 : 3;
  p.b_kmajor = b_kmajor;
  p.dbg = dbg;

  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= kMaxDevices) return set_error("device ordinal out of range"), NU_EINVAL;
  static std::atomic<int> num_sms[kMaxDevices];
  static std::atomic<int> configured[kMaxDevices];
  if (num_sms[dev].load() == 0) {
    int n = 0;
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    num_sms[dev].store(n > 0 ? n : 148);
  }
  if (!configured[dev].load()) {
    cudaError_t e = cudaFuncSetAttribute(leaf_gemm_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return set_error("cudaFuncSetAttribute: %s", cudaGetErrorString(e)), NU_ECUDA;
    configured[dev].store(1);
  }
  const int tiles = p.tiles_m * p.tiles_n;
  const int sms = num_sms[dev].load();
  const int grid = tiles < sms ? tiles : sms;
  leaf_gemm_kernel<<<grid, NUM_THREADS, SMEM_BYTES, stream>>>(tmA, tmB, p);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_error("leaf launch: %s", cudaGetErrorString(e)), NU_ECUDA;
  return 0;
}

}  // namespace nu

// Debug entry (not part of northup.h): B K-major variant and a stage dump.
extern "C" int northup_debug_leaf_gemm(const float* A, int64_t lda, const float* B, int64_t ldb,
                                       float* C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                                       int accumulate, int64_t kc, int npass, int b_kmajor,
                                       float* dbg, void* stream) {
  return nu::leaf_gemm_launch_dbg(A, lda, B, ldb, C, ldc, M, N, K, accumulate, kc, npass, b_kmajor,
                                  dbg, static_cast<cudaStream_t>(stream));
}
