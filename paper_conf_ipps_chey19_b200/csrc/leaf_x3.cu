// The leaf (S§8 a5-a7): C (+)= A.B for one K panel on the split operands of
// split.cu (reading R22), as a CTA pair (cluster of 2 on one
// TPC, tcgen05.mma.cta_group::2, pair tile 256 x 256).
//
//   * TMA (SW128) streams per 32-k stage A' (128 rows x [hi 32 | lo 32] fp16,
//     16 KiB) and B' (64 rows [hi 16; lo 16; hi 16; lo 16] x 128 n fp16,
//     16 KiB) into a STAGES-deep ring in each CTA; both CTAs' loads complete
//     on the leader's barrier (.cta_group::2).
//   * The leader's MMA thread issues per 16 k three kind::f16 MMAs (fp16 in,
//     fp32 accumulate, M 256 N 256 K 16): hi.hi, hi.lo, lo.hi.
//   * The tensor core truncates its fp32 accumulator after every MMA (probed,
//     DESIGN.md R20), so the accumulation runs in TMEM for kAccChunk (256) of
//     K only; two 256-column accumulators alternate, so the epilogue drains
//     one while the MMAs fill the other.
//   * Epilogue (16 warps, four per TMEM lane quarter): each thread owns one row
//     and 64 columns of its CTA's half tile and adds every chunk into a running
//     sum in registers (fp32 round-to-nearest, ascending K).  At the end
//     of the panel it scales by 2^(e_i + e_j) (exact) and writes C once through
//     a 128-B-swizzled 32 x 32 staging box (8 boxes, shared by warps w and
//     w + 8 in turn): a TMA store, or a TMA reduce-add (C += panel, an fp32 RN
//     add in L2) when accumulating.  A C that TMA cannot address (unaligned)
//     is written from registers.
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <string.h>

#include <algorithm>
#include <atomic>

#include "leaf_common.cuh"
#include "northup_internal.h"

namespace nu {
namespace leaf {
namespace x3 {

constexpr int BM = 256, BN = 256, BM_CTA = 128, BN_CTA = 128;
constexpr int KS = 32;                               // real k per stage
constexpr int STAGES = 6;

constexpr int A_BYTES = BM_CTA * 2 * KS * 2;         // 16 KiB
constexpr int B_HALF_BYTES = 2 * KS * 64 * 2;        // 64 rows x 64 n fp16 = 8 KiB
constexpr int B_BYTES = 2 * B_HALF_BYTES;            // 16 KiB
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int EPI_WARP0 = 2;
constexpr int EPI_WARPS = 16;                         // four per TMEM lane quarter, 64 columns each
constexpr int EPI_THREADS = 32 * EPI_WARPS;
constexpr int EPI_COLS = 64;                          // tile columns per epilogue thread (its running sum)
constexpr int BOX_BYTES = 32 * 32 * 4;                // one staging box: 32 rows x 32 fp32
constexpr int EPI_BOXES = EPI_WARPS / 2;               // shared by warps ew and ew + 8, in turn
constexpr int EPI_BYTES = EPI_BOXES * BOX_BYTES;
constexpr int NUM_THREADS = 32 * (EPI_WARP0 + EPI_WARPS);
constexpr int TMEM_COLS = 512;                       // two 256-column accumulators
constexpr int BAR_BYTES = 256;
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + EPI_BYTES + BAR_BYTES + 1024;
static_assert(SMEM_BYTES <= 227 * 1024, "shared memory budget");

struct Params {
  float* C;
  int64_t ldc;
  const int* ea;   // row exponents (M)
  const int* eb;   // column exponents (N)
  int M, N, Kp;    // Kp: panel K rounded up to KS (the split zero-pads)
  int kb_per_chunk;   // stages per TMEM accumulation chunk
  int accumulate;     // 1: C += A.B (the epilogue's write is a TMA reduce-add)
  int tiles_m, tiles_n, band;
  int vec_ok;      // C 16-B aligned with ldc % 4 == 0: TMA epilogue
  int npass;       // 1: hi.hi only (negative test), 3: product, 4: + lo.lo
  float* dbg;      // profile mode: per-cluster cycle counters (NULL in production)
};

__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t mapa(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint32_t bar, uint32_t parity) {
  uint32_t done = 0;
  uint64_t t0 = 0;
  for (uint32_t it = 0;; ++it) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
    if (done) return;
    if ((it & 1023u) == 0) {
      const uint64_t t = globaltimer();
      if (it == 0) t0 = t;
      else if (t - t0 > 4000000000ull) __trap();   // a broken invariant traps instead of hanging
    }
  }
}
// TMA load into this CTA's shared memory; the bytes complete on `bar`, which
// may be the leader CTA's barrier (cta_group::2).
__device__ __forceinline__ void tma_load_pair(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0,
                                              int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.cta_group::2"
      " [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void tma_load_pair_4d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0,
                                                 int c1, int c2, int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes.cta_group::2"
      " [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void umma_f16_pair(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc,
                                              uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(da), "l"(db), "r"(idesc), "r"(accum)
      : "memory");
}
// Arrive on the same barrier offset in both CTAs once the MMAs issued so far completed.
__device__ __forceinline__ void umma_commit_pair(uint32_t bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64"
      " [%0], %1;" ::"r"(bar),
      "h"(static_cast<uint16_t>(3))
      : "memory");
}
// kind::f16 instruction descriptor: D f32 [4,6)=1, A fp16 [7,10)=0, B fp16
// [10,13)=0, A K-major [15]=0, B MN-major [16]=1, N>>3 [17,23), M>>4 [24,29).
__host__ __device__ constexpr uint32_t idesc_f16(int m, int n) {
  return (1u << 4) | (0u << 7) | (0u << 10) | (0u << 15) | (1u << 16) |
         (static_cast<uint32_t>(n >> 3) << 17) | (static_cast<uint32_t>(m >> 4) << 24);
}
__device__ __forceinline__ void sts128(uint32_t a, uint32_t x, uint32_t y, uint32_t z, uint32_t w) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(x), "r"(y), "r"(z), "r"(w)
               : "memory");
}
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(src), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void tma_reduce_add_2d(const CUtensorMap* map, uint32_t src, int c0, int c1) {
  asm volatile("cp.reduce.async.bulk.tensor.2d.global.shared::cta.add.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(src), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t count) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// v * 2^e for |e| <= 252 (two exact power-of-two factors, each a normal float).
__device__ __forceinline__ float scale2(float v, int e) {
  const int e1 = e >> 1, e2 = e - e1;
  return v * __uint_as_float(static_cast<uint32_t>(e1 + 127) << 23) *
         __uint_as_float(static_cast<uint32_t>(e2 + 127) << 23);
}

// TMEM -> registers, 16 columns of this warp's lane quarter.
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(NUM_THREADS, 1)
    leaf_x3_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmC, const Params p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  uint8_t* epi_base = smem + STAGES * STAGE_BYTES;
  uint8_t* bars = epi_base + EPI_BYTES;
  const uint32_t bar_full = smem_u32(bars);             // [STAGES] leader: both CTAs' bytes landed
  const uint32_t bar_empty = bar_full + 8 * STAGES;     // [STAGES] each CTA: stage consumed
  const uint32_t bar_tfull = bar_empty + 8 * STAGES;    // [2] each CTA: accumulator ready
  const uint32_t bar_tempty = bar_tfull + 16;           // [2] leader: accumulator drained
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 8 * (2 * STAGES + 4));

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;

  if (threadIdx.x == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    if (p.vec_ok) prefetch_tmap(&tmC);
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(bar_full + 8 * s, 1);
      mbar_init(bar_empty + 8 * s, 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(bar_tfull + 8 * b, 1);
      mbar_init(bar_tempty + 8 * b, 2 * EPI_THREADS);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
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
  const int nkb = p.Kp / KS;
  const int nchunks = (nkb + p.kb_per_chunk - 1) / p.kb_per_chunk;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      const uint32_t full_leader = mapa(bar_full, 0);
      uint32_t it = 0;
      for (int t = cid; t < num_tiles; t += nclusters) {
        int mb, nb;
        tile_coords(t, p.tiles_m, p.tiles_n, p.band, mb, nb);
        const int row0 = mb * BM + rank * BM_CTA;
        const int col0 = nb * BN + rank * BN_CTA;
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const uint32_t s = it % STAGES, use = it / STAGES;
          mbar_wait(bar_empty + 8 * s, (use & 1) ^ 1);
          if (leader) mbar_arrive_expect_tx(bar_full + 8 * s, 2 * STAGE_BYTES);
          const uint32_t sa = smem_u32(smem + s * STAGE_BYTES);
          const uint32_t fb = full_leader + 8 * s;
          tma_load_pair(sa, &tmA, fb, kb * 2 * KS, row0);
          // B' box (64 n, 16 k, hi/lo, 2 k-groups) lands as rows 32 g + 16 part + k
          tma_load_pair_4d(sa + A_BYTES, &tmB, fb, col0, 0, 0, 2 * kb);
          tma_load_pair_4d(sa + A_BYTES + B_HALF_BYTES, &tmB, fb, col0 + 64, 0, 0, 2 * kb);
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer (leader CTA)
    if (leader && lane == 0) {
      const uint32_t idesc = idesc_f16(BM, BN);
      uint32_t it = 0, chunk_it = 0;
      long long w_full = 0, w_te = 0;
      const long long t_beg = clock64();
      for (int t = cid; t < num_tiles; t += nclusters) {
        for (int ch = 0; ch < nchunks; ++ch, ++chunk_it) {
          const uint32_t b = chunk_it & 1;
          long long c0 = clock64();
          mbar_wait_cluster(bar_tempty + 8 * b, ((chunk_it >> 1) & 1) ^ 1);
          w_te += clock64() - c0;
          tc_fence_after();
          const uint32_t d = tmem_base + 256 * b;
          const int kb0 = ch * p.kb_per_chunk;
          const int kb1 = min(nkb, kb0 + p.kb_per_chunk);
          uint32_t acc = 0;
          for (int kb = kb0; kb < kb1; ++kb, ++it) {
            const uint32_t s = it % STAGES, use = it / STAGES;
            c0 = clock64();
            mbar_wait(bar_full + 8 * s, use & 1);
            w_full += clock64() - c0;
            tc_fence_after();
            const uint32_t sa = smem_u32(smem + s * STAGE_BYTES);
            const uint32_t sb = sa + A_BYTES;
#pragma unroll
            for (int g = 0; g < 2; ++g) {
              const uint64_t a_hi = umma_desc(sa + 32 * g, 16, 1024);
              const uint64_t a_lo = umma_desc(sa + 64 + 32 * g, 16, 1024);
              const uint64_t b_hi = umma_desc(sb + (2 * g) * 2048, B_HALF_BYTES, 1024);
              const uint64_t b_lo = umma_desc(sb + (2 * g + 1) * 2048, B_HALF_BYTES, 1024);
              umma_f16_pair(d, a_hi, b_hi, idesc, acc);
              acc = 1;
              if (p.npass >= 3) {
                umma_f16_pair(d, a_hi, b_lo, idesc, 1u);
                umma_f16_pair(d, a_lo, b_hi, idesc, 1u);
              }
              if (p.npass >= 4) umma_f16_pair(d, a_lo, b_lo, idesc, 1u);
            }
            umma_commit_pair(bar_empty + 8 * s);
          }
          umma_commit_pair(bar_tfull + 8 * b);
        }
      }
      if (p.dbg) {
        float* o = p.dbg + 4 * cid;
        o[0] = static_cast<float>(clock64() - t_beg);
        o[1] = static_cast<float>(w_full);
        o[2] = static_cast<float>(w_te);
        o[3] = static_cast<float>(it);
      }
    }
  } else {
    // ---------------------------------------------------- epilogue (own rows)
    // Thread (quarter q, lane) owns row 32 q + lane of this CTA's half of the
    // tile and columns [64 cg, 64 cg + 64): it adds every chunk's accumulator
    // into a running fp32 sum (round-to-nearest, in ascending chunk order,
    // P:299) and writes the tile once, scaled by 2^(e_i + e_j).
    const int ew = warp - EPI_WARP0;
    const int q = warp & 3;                                   // TMEM lane quarter
    const int cg = ew >> 2;                                   // 64-column group
    const uint32_t tempty_leader = mapa(bar_tempty, 0);
    const uint32_t box = smem_u32(epi_base + (ew % EPI_BOXES) * BOX_BYTES);
    const uint32_t t_row = tmem_base + (static_cast<uint32_t>(32 * q) << 16) + EPI_COLS * cg;
    uint32_t chunk_it = 0;
    for (int t = cid; t < num_tiles; t += nclusters) {
      int mb, nb;
      tile_coords(t, p.tiles_m, p.tiles_n, p.band, mb, nb);
      const int row0 = mb * BM + rank * BM_CTA + 32 * q;     // this warp's 32 rows
      const int grow = row0 + lane;
      float sum[EPI_COLS];
#pragma unroll
      for (int j = 0; j < EPI_COLS; ++j) sum[j] = 0.f;
      for (int ch = 0; ch < nchunks; ++ch, ++chunk_it) {
        const uint32_t b = chunk_it & 1;
        mbar_wait(bar_tfull + 8 * b, (chunk_it >> 1) & 1);
        tc_fence_after();
#pragma unroll
        for (int pc = 0; pc < EPI_COLS / 16; ++pc) {
          uint32_t v[16];
          tmem_ld16(t_row + 256 * b + 16 * pc, v);
#pragma unroll
          for (int j = 0; j < 16; ++j) sum[16 * pc + j] = __fadd_rn(sum[16 * pc + j], __uint_as_float(v[j]));
        }
        tc_fence_before();
        mbar_arrive_cluster(tempty_leader + 8 * b);         // accumulator b is free again
      }
      const int er = grow < p.M ? p.ea[grow] : 0;
#pragma unroll
      for (int h = 0; h < EPI_COLS / 32; ++h) {      // scale by 2^(e_i + e_j), in place
        const int gcol0 = nb * BN + EPI_COLS * cg + 32 * h;
        const int ebl = (gcol0 + lane < p.N) ? p.eb[gcol0 + lane] : 0;
#pragma unroll
        for (int j = 0; j < 32; ++j) sum[32 * h + j] = scale2(sum[32 * h + j], er + __shfl_sync(0xffffffffu, ebl, j));
      }
      // write the tile: warps ew < 8 first, then warps ew >= 8 reuse their boxes
#pragma unroll
      for (int turn = 0; turn < 2; ++turn) {
        if ((ew >> 3) == turn) {
#pragma unroll
          for (int h = 0; h < EPI_COLS / 32; ++h) {
            const int gcol0 = nb * BN + EPI_COLS * cg + 32 * h;
            const float* v = sum + 32 * h;
            if (p.vec_ok) {
              if (lane == 0) bulk_wait_read<0>();             // the box's previous store has read it
              __syncwarp();
              const uint32_t rowp = box + lane * 128;
#pragma unroll
              for (int i = 0; i < 8; ++i)
                sts128(rowp + ((i ^ (lane & 7)) << 4), __float_as_uint(v[4 * i]), __float_as_uint(v[4 * i + 1]),
                       __float_as_uint(v[4 * i + 2]), __float_as_uint(v[4 * i + 3]));
              fence_proxy_async_smem();
              __syncwarp();
              if (lane == 0) {
                if (p.accumulate) tma_reduce_add_2d(&tmC, box, gcol0, row0);
                else tma_store_2d(&tmC, box, gcol0, row0);
                bulk_commit();
              }
            } else if (grow < p.M) {
              float* dst = p.C + static_cast<int64_t>(grow) * p.ldc + gcol0;
#pragma unroll
              for (int j = 0; j < 32; ++j) {
                if (gcol0 + j >= p.N) continue;
                dst[j] = p.accumulate ? __fadd_rn(dst[j], v[j]) : v[j];
              }
            }
          }
          if (lane == 0) bulk_wait_read<0>();                 // boxes free for the other turn
          __syncwarp();
        }
        named_bar_sync(2, EPI_THREADS);
      }
    }
    if (lane == 0) bulk_wait_all();
  }

  tc_fence_before();
  __syncthreads();
  cluster_sync();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(TMEM_COLS)
                 : "memory");
  }
}

}  // namespace x3

void preload_x3() {
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, x3::leaf_x3_kernel);
  preload_split();
}

// The GEMM of one K panel on split operands (split.cu layouts).
int x3_gemm(const SplitOperand& A, const SplitOperand& B, float* C, int64_t ldc, int m, int n, int kl,
            int accumulate, int kb_per_chunk, int npass, int band, int sms, int dev, float* dbg,
            cudaStream_t stream) {
  using namespace x3;
  const int Kp = (kl + KS - 1) / KS * KS;
  int rc;
  CUtensorMap tmA, tmB, tmC;
  {
    const cuuint64_t dims[2] = {2 * static_cast<cuuint64_t>(Kp), static_cast<cuuint64_t>(m)};
    const cuuint64_t strides[1] = {4 * static_cast<cuuint64_t>(A.ld)};
    const cuuint32_t box[2] = {64, BM_CTA};
    if ((rc = encode_tiled(&tmA, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, A.p, dims, strides, box,
                           CU_TENSOR_MAP_SWIZZLE_128B)))
      return rc;
  }
  {
    const cuuint64_t dims[4] = {static_cast<cuuint64_t>(n), 16, 2, static_cast<cuuint64_t>(Kp / 16)};
    const cuuint64_t strides[3] = {4 * static_cast<cuuint64_t>(B.ld), 2 * static_cast<cuuint64_t>(B.ld),
                                   64 * static_cast<cuuint64_t>(B.ld)};
    const cuuint32_t box[4] = {64, 16, 2, 2};
    if ((rc = encode_tiled(&tmB, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, B.p, dims, strides, box,
                           CU_TENSOR_MAP_SWIZZLE_128B)))
      return rc;
  }
  x3::Params p;
  p.C = C;
  p.ldc = ldc;
  p.ea = A.e;
  p.eb = B.e;
  p.M = m;
  p.N = n;
  p.Kp = Kp;
  p.kb_per_chunk = kb_per_chunk;
  p.accumulate = accumulate;
  p.tiles_m = (m + BM - 1) / BM;
  p.tiles_n = (n + BN - 1) / BN;
  p.band = band;
  p.vec_ok = (reinterpret_cast<uintptr_t>(C) % 16 == 0) && (ldc % 4 == 0);
  p.npass = npass;
  p.dbg = dbg;
  if (p.vec_ok) {
    if ((rc = encode_2d(&tmC, C, n, m, ldc, 32, 32))) return rc;
  } else {
    memset(&tmC, 0, sizeof(tmC));
  }
  static std::atomic<int> configured[kMaxDevices];
  if (!configured[dev].load()) {
    cudaError_t e = cudaFuncSetAttribute(leaf_x3_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return fail(NU_ECUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(e));
    configured[dev].store(1);
  }
  const int tiles = p.tiles_m * p.tiles_n;
  const int pairs = sms / 2;
  const int grid = 2 * (tiles < pairs ? tiles : pairs);
  leaf_x3_kernel<<<grid, NUM_THREADS, SMEM_BYTES, stream>>>(tmA, tmB, tmC, p);
  count_launches(1);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : fail(NU_ECUDA, "leaf launch: %s", cudaGetErrorString(e));
}

}  // namespace leaf
}  // namespace nu
