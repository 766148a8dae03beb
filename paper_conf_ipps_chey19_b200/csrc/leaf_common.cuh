// Shared device-side helpers of the sm_100a leaf kernels: mbarriers, TMA,
// tcgen05 (UMMA descriptors, MMA, commit, TMEM loads) and tile rasterisation.
#pragma once

#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace nu {
namespace leaf {

constexpr int UMMA_K = 8;            // K per tcgen05.mma kind::tf32
constexpr int BK = 32;               // K elements per pipeline stage (128-B rows)
constexpr int B_CHUNK = 32;          // N columns per 128-B swizzle atom
constexpr int B_CHUNK_BYTES = B_CHUNK * BK * 4;    // 4 KiB: one TMA box of B

// Kernel parameters shared by the leaf variants.
struct Params {
  float* C;
  int64_t ldc;
  int M, N, K;
  int kb_per_chunk;   // k-blocks (of BK) per TMEM accumulation chunk
  int accumulate;     // 1: C += A.B ; 0: C = A.B
  int tiles_m, tiles_n;
  int vec_ok;         // C base and ldc allow 16-byte vector access
  int band;           // n-blocks per raster band (L2 reuse across concurrent tiles)
  int npass;          // 3 = 3xTF32 (product path), 1 = plain TF32 (negative test)
  int b_kmajor;       // debug: B given as N x K (K-major) instead of K x N
  float* dbg;         // debug: dump of stage 0 after the split (NULL in production)
  const float* A;     // operands for the LDG-fed kernel (v2): row-major, 16-B aligned
  int64_t lda;
  const float* B;
  int64_t ldb;
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

struct LaunchArgs {
  const float* A;
  int64_t lda;
  const float* B;
  int64_t ldb;
  Params p;
  cudaStream_t stream;
  int dev;
  int sms;
};

// cuTensorMapEncodeTiled for a row-major fp32 matrix viewed as (inner, outer).
int encode_2d(CUtensorMap* map, const float* base, uint64_t inner, uint64_t outer,
              uint64_t ld_elems, uint32_t box_inner, uint32_t box_outer,
              CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B);
int encode_2d_bf16(CUtensorMap* map, const void* base, uint64_t inner, uint64_t outer, uint64_t ld_elems,
                   uint32_t box_inner, uint32_t box_outer);
int launch_sm1(LaunchArgs& a);   // v0: 1-CTA 128 x 256 tile
int launch_sm2(LaunchArgs& a);   // v1: CTA pair (cta_group::2) 256 x 256 tile, TMA-fed
int launch_sm3(LaunchArgs& a);   // v2: CTA pair, split warps load global memory directly
int launch_sm4(LaunchArgs& a);   // v3: CTA pair, A' operand in TMEM, TMA-store epilogue
// Load each variant's kernel now (lazy module loading would otherwise load it at its
// first launch, which can block behind a stream that waits on another process).
void preload_sm1();
void preload_sm2();
void preload_sm3();
void preload_sm4();
bool launch_sm4_ok(const LaunchArgs& a);

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
int64_t split_b_max_n();
void preload_split();
void preload_x3();
// GEMM of one K panel (kl <= the panel) on split operands.
int x3_gemm(const SplitOperand& A, const SplitOperand& B, float* C, int64_t ldc, int m, int n, int kl,
            int accumulate, int kb_per_chunk, int npass, int band, int sms, int dev, float* dbg,
            cudaStream_t stream);

}  // namespace leaf
}  // namespace nu
