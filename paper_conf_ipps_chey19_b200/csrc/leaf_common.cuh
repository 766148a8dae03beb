// Device-side helpers of the sm_100a leaf (leaf_x3.cu): mbarriers, TMA,
// UMMA shared-memory descriptors and tile rasterisation; host-side
// declarations of the split (split.cu) and the GEMM launch.
#pragma once

#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace nu {
namespace leaf {

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
//   2 = SWIZZLE_128B (16-B granules XOR row%8; K-major A, and MN-major 16-bit B
//       with LBO = the stride between 64-element MN atoms).
constexpr uint32_t LAYOUT_SW128 = 2;
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

// Tile t -> (m-block, n-block): bands of `band` n-blocks, m fastest inside a
// band, so the tiles in flight at one time share `band` B strips and a short
// run of A strips in L2.
__device__ __forceinline__ void tile_coords(int t, int tiles_m, int tiles_n, int band_w, int& mb,
                                            int& nb) {
  const int band = t / (tiles_m * band_w);
  const int rem = t - band * tiles_m * band_w;
  const int n0 = band * band_w;
  const int bw = min(band_w, tiles_n - n0);
  mb = rem / bw;
  nb = n0 + rem % bw;
}

}  // namespace leaf
}  // namespace nu

// ------------------------------------------------------------- host side
namespace nu {
namespace leaf {

// cuTensorMapEncodeTiled for a row-major fp32 matrix viewed as (inner, outer).
int encode_2d(CUtensorMap* map, const float* base, uint64_t inner, uint64_t outer,
              uint64_t ld_elems, uint32_t box_inner, uint32_t box_outer,
              CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B);
// cuTensorMapEncodeTiled, general rank (strides in bytes for dims 1..rank-1).
int encode_tiled(CUtensorMap* map, CUtensorMapDataType type, int rank, const void* base,
                 const cuuint64_t* dims, const cuuint64_t* strides, const cuuint32_t* box,
                 CUtensorMapSwizzle swz);

// A split operand (split.cu, R22): `p` holds the hi/lo fp16 pairs in
// the layout of a row-major fp32 matrix with leading dimension `ld` (floats),
// `e` one exponent per row (A) or column (B) of the panel.
struct SplitOperand {
  const float* p;
  int64_t ld;
  const int* e;
};
int split_a_launch(const float* A, int64_t lda, int M, int Kl, float* dst, int64_t ldd, int* ea, int sms,
                   cudaStream_t s);
int split_b_launch(const float* B, int64_t ldb, int Kl, int N, float* dst, int64_t ldd, int* eb,
                   unsigned* bmax, cudaStream_t s);
// Both splits of a small panel in one launch (B out of place); see kSplitSmall.
int split_ab_small_launch(const float* A, int64_t lda, int M, int Kl, float* adst, int64_t ldda, int* ea,
                          const float* B, int64_t ldb, int N, float* bdst, int64_t lddb, int* eb, cudaStream_t s);
int64_t split_b_max_n();
void preload_split();
void preload_x3();
// GEMM of one K panel (kl <= the panel) on split operands.
int x3_gemm(const SplitOperand& A, const SplitOperand& B, float* C, int64_t ldc, int m, int n, int kl,
            int accumulate, int kb_per_chunk, int npass, int band, int sms, int dev, float* dbg,
            cudaStream_t stream);

}  // namespace leaf
}  // namespace nu
