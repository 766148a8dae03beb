// Host side of the leaf: TMA descriptor encoding, argument validation and
// dispatch between the leaf kernel variants.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <atomic>

#include "leaf_common.cuh"
#include "northup_internal.h"

namespace nu {
namespace leaf {

static PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

static int get_encode() {
  if (g_encode) return 0;
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaError_t e = cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fn, 12000,
                                                   cudaEnableDefault, &q);
  if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
    return fail(NU_ECUDA, "cuTensorMapEncodeTiled unavailable: %s", cudaGetErrorString(e));
  g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  return 0;
}

int encode_2d(CUtensorMap* map, const float* base, uint64_t inner, uint64_t outer,
              uint64_t ld_elems, uint32_t box_inner, uint32_t box_outer, CUtensorMapSwizzle swz) {
  int rc = get_encode();
  if (rc) return rc;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {ld_elems * 4};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = g_encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims,
                        strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS)
    return fail(NU_EINVAL, "cuTensorMapEncodeTiled failed (%d): base=%p inner=%llu outer=%llu ld=%llu",
                (int)r, (const void*)base, (unsigned long long)inner, (unsigned long long)outer,
                (unsigned long long)ld_elems);
  return 0;
}

// bf16 2-D map with 128-B swizzle (the pre-split operands of NU_LEAF2_PRESPLIT).
int encode_2d_bf16(CUtensorMap* map, const void* base, uint64_t inner, uint64_t outer, uint64_t ld_elems,
                   uint32_t box_inner, uint32_t box_outer) {
  int rc = get_encode();
  if (rc) return rc;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {ld_elems * 2};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = g_encode(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box,
                        estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? 0 : fail(NU_EINVAL, "cuTensorMapEncodeTiled (bf16) failed (%d)", (int)r);
}

}  // namespace leaf

int default_leaf_variant() {
  static int env_variant = -1;
  if (env_variant < 0) {
    const char* v = getenv("NORTHUP_LEAF");
    env_variant = (v && v[0] >= '1' && v[0] <= '4') ? v[0] - '0' : kDefaultLeafVariant;
  }
  return env_variant;
}

// Test hook (NORTHUP_DEBUG_SLOW_SIBLING="w,pct", exec.cpp): a one-thread kernel
// that holds a stream for `ns` nanoseconds, emulating a slower sibling.
__global__ void debug_spin_kernel(long long ns) {
  const long long t0 = clock64();
  const long long cycles = ns * 2;   // ~2 GHz
  while (clock64() - t0 < cycles) __nanosleep(1000);
}

// Multi-process siblings (peer.cpp): store a generation into a flag word that
// may live in another process's (and another GPU's) memory, after everything
// earlier on the stream.  A one-thread kernel with a system-scope release store
// works for any peer-mapped address, where a stream memory operation on peer
// memory is not guaranteed to.
__global__ void flag_store_kernel(uint32_t* addr, uint32_t v) {
  __threadfence_system();
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(addr), "r"(v) : "memory");
}

int flag_store_launch(uint32_t* addr, uint32_t v, cudaStream_t s) {
  flag_store_kernel<<<1, 1, 0, s>>>(addr, v);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : cuda_fail(e, "flag_store_kernel");
}

// Load every kernel the executor may launch on the current device (see
// leaf_common.cuh preload_sm*): run before work that waits on other processes.
void preload_kernels() {
  leaf::preload_sm1();
  leaf::preload_sm2();
  leaf::preload_sm3();
  leaf::preload_sm4();
  hotspot_preload();
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, debug_spin_kernel);
  cudaFuncGetAttributes(&fa, flag_store_kernel);
}

int debug_spin(long long ns, cudaStream_t s) {
  debug_spin_kernel<<<1, 1, 0, s>>>(ns);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : cuda_fail(e, "debug_spin_kernel");
}

int debug_slow_sibling(int* us) {
  int w = -1, t = 0;
  if (const char* e = getenv("NORTHUP_DEBUG_SLOW_SIBLING")) sscanf(e, "%d,%d", &w, &t);
  *us = t;
  return w;
}

bool leaf_tma_legal(const void* p, int64_t ld) {
  return (reinterpret_cast<uintptr_t>(p) % 16 == 0) && (ld % 4 == 0) && ld > 0;
}

// variant: 0 = default (env NORTHUP_LEAF=1..4 may override), 1 = v0 (1 CTA), 2 = v1.2 (pair),
// 3 = v2 (pair, LDG-fed), 4 = v3 (pair, A' in TMEM).
int leaf_gemm_launch_dbg(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                         int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t kc,
                         int npass, int b_kmajor, float* dbg, int variant, cudaStream_t stream) {
  using namespace leaf;
  if (M < 0 || N < 0 || K < 0) return fail(NU_EINVAL, "negative dimension");
  if (M == 0 || N == 0) return 0;
  if (K == 0) {
    if (accumulate) return 0;
    cudaError_t e = cudaMemset2DAsync(C, ldc * 4, 0, N * 4, M, stream);
    return e == cudaSuccess ? 0 : fail(NU_ECUDA, "memset: %s", cudaGetErrorString(e));
  }
  if (M > INT32_MAX || N > INT32_MAX || K > INT32_MAX)
    return fail(NU_EINVAL, "dimension exceeds int32 TMA coordinates");
  if (!leaf_tma_legal(A, lda) || !leaf_tma_legal(B, ldb))
    return fail(NU_EINVAL, "leaf operands need 16-B aligned base and ld %% 4 == 0");
  if (lda < K || ldb < (b_kmajor ? K : N) || ldc < N) return fail(NU_EINVAL, "leading dimension too small");
  if (kc <= 0) kc = K;
  if (kc % BK) kc = (kc + BK - 1) / BK * BK;   // chunks are whole k-blocks
  int64_t kbpc = (kc + BK - 1) / BK;
  if (kbpc < 1) kbpc = 1;
  if (kbpc > INT32_MAX) kbpc = INT32_MAX;

  LaunchArgs a;
  a.A = A;
  a.lda = lda;
  a.B = B;
  a.ldb = ldb;
  a.stream = stream;
  Params& p = a.p;
  p.C = C;
  p.ldc = ldc;
  p.M = static_cast<int>(M);
  p.N = static_cast<int>(N);
  p.K = static_cast<int>(K);
  p.kb_per_chunk = static_cast<int>(kbpc);
  p.accumulate = accumulate ? 1 : 0;
  p.vec_ok = (reinterpret_cast<uintptr_t>(C) % 16 == 0) && (ldc % 4 == 0);
  p.npass = (npass == 1 || npass == 2) ? npass : (npass == 3 ? 3 : kDefaultNpass);
  p.b_kmajor = b_kmajor;
  p.dbg = dbg;
  p.tiles_m = p.tiles_n = 0;
  static int env_band = -1;
  if (env_band < 0) {
    const char* v = getenv("NORTHUP_RASTER_BAND");
    env_band = (v && atoi(v) > 0) ? atoi(v) : kRasterBand;
  }
  p.band = env_band;

  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= kMaxDevices) return fail(NU_EINVAL, "device ordinal out of range");
  static std::atomic<int> num_sms[kMaxDevices];
  if (num_sms[dev].load() == 0) {
    int n = 0;
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    num_sms[dev].store(n > 0 ? n : 148);
  }
  a.dev = dev;
  a.sms = num_sms[dev].load();
  if (variant == 0) variant = default_leaf_variant();
  if (variant == 1 && p.npass == 2) p.npass = 3;   // the 1-CTA v0 kernel has no bf16 path
  if (variant == 3 && (p.npass != 2 || b_kmajor)) variant = 2;   // v2 implements R21 only
  // K-panel launches: each launch covers `panel` of K for
  // every tile, so all CTAs stream the same K range and share A/B panels in
  // L2; the grid-wide launch boundary re-synchronises them.  panel is a
  // multiple of k_chunk, so results are bitwise those of a single launch.
  static int64_t env_panel = -1;
  if (env_panel < 0) {
    const char* v = getenv("NORTHUP_PANEL_CHUNKS");
    env_panel = (v && atoll(v) >= 0) ? atoll(v) : kPanelChunks;
  }
  const int64_t panel = env_panel > 0 ? env_panel * kbpc * BK : K;
  int rc = 0;
  for (int64_t k0 = 0; k0 < K && rc == 0; k0 += panel) {
    LaunchArgs b = a;
    const int64_t kk = K - k0 < panel ? K - k0 : panel;
    b.A = A + k0;
    b.B = B + (b_kmajor ? k0 : k0 * ldb);
    b.p.K = static_cast<int>(kk);
    b.p.accumulate = (k0 > 0 || accumulate) ? 1 : 0;
    b.p.A = b.A;
    b.p.lda = lda;
    b.p.B = b.B;
    b.p.ldb = ldb;
    if (variant == 4 && !launch_sm4_ok(b)) variant = 2;
    rc = variant == 1 ? launch_sm1(b) : variant == 3 ? launch_sm3(b) : variant == 4 ? launch_sm4(b) : launch_sm2(b);
  }
  return rc;
}

int leaf_gemm_launch(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                     int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t kc,
                     int npass, cudaStream_t stream) {
  return leaf_gemm_launch_dbg(A, lda, B, ldb, C, ldc, M, N, K, accumulate, kc, npass, 0, nullptr, 0,
                              stream);
}

}  // namespace nu

// Debug entry (not part of northup.h): the leaf variant default calls use.
extern "C" int northup_debug_leaf_variant(void) { return nu::default_leaf_variant(); }

// Debug entry (not part of northup.h): kernel variant, B K-major, stage dump.
extern "C" int northup_debug_leaf_gemm(const float* A, int64_t lda, const float* B, int64_t ldb,
                                       float* C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                                       int accumulate, int64_t kc, int npass, int b_kmajor,
                                       float* dbg, int variant, void* stream) {
  return nu::leaf_gemm_launch_dbg(A, lda, B, ldb, C, ldc, M, N, K, accumulate, kc, npass, b_kmajor,
                                  dbg, variant, static_cast<cudaStream_t>(stream));
}
