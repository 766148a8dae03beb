// Host side of the leaf: TMA descriptor encoding, argument validation and
// dispatch between the leaf kernel variants.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <atomic>
#include <mutex>

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

int encode_tiled(CUtensorMap* map, CUtensorMapDataType type, int rank, const void* base, const cuuint64_t* dims,
                 const cuuint64_t* strides, const cuuint32_t* box, CUtensorMapSwizzle swz) {
  int rc = get_encode();
  if (rc) return rc;
  cuuint32_t estr[5] = {1, 1, 1, 1, 1};
  CUresult r = g_encode(map, type, rank, const_cast<void*>(base), dims, strides, box, estr,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS)
    return fail(NU_EINVAL, "cuTensorMapEncodeTiled (rank %d) failed (%d): base=%p dim0=%llu", rank, (int)r, base,
                (unsigned long long)dims[0]);
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
    env_variant = (v && v[0] >= '1' && v[0] <= '5') ? v[0] - '0' : kDefaultLeafVariant;
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
  leaf::preload_x3();
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

// ------------------------------------------------------------------ the x3 leaf
// Stream-ordered scratch for leaf calls that bring none (northup_leaf_gemm):
// a private pool per device that keeps its memory (no release at syncs).
static std::mutex g_pool_mu;
static cudaMemPool_t g_pool[kMaxDevices];

static int scratch_alloc(int dev, uint64_t bytes, cudaStream_t s, char** out) {
  {
    std::lock_guard<std::mutex> g(g_pool_mu);
    if (!g_pool[dev]) {
      cudaMemPoolProps pr = {};
      pr.allocType = cudaMemAllocationTypePinned;
      pr.handleTypes = cudaMemHandleTypeNone;
      pr.location.type = cudaMemLocationTypeDevice;
      pr.location.id = dev;
      cudaError_t e = cudaMemPoolCreate(&g_pool[dev], &pr);
      if (e != cudaSuccess) return cuda_fail(e, "cudaMemPoolCreate (leaf scratch)");
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(g_pool[dev], cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  cudaError_t e = cudaMallocFromPoolAsync(reinterpret_cast<void**>(out), bytes, g_pool[dev], s);
  return e == cudaSuccess ? 0 : fail(NU_ENOMEM, "leaf scratch (%llu B): %s", (unsigned long long)bytes,
                                     cudaGetErrorString(e));
}

static inline uint64_t al256(uint64_t b) { return (b + 255) / 256 * 256; }

uint64_t leaf_scratch_bytes(int64_t m, int64_t n, int64_t panel, bool b_presplit) {
  const uint64_t Kp = static_cast<uint64_t>((panel + 31) / 32 * 32);
  uint64_t s = al256(4ull * m * Kp) + al256(4ull * m);
  if (!b_presplit) s += al256(4ull * Kp * static_cast<uint64_t>((n + 31) / 32 * 32)) + 2 * al256(4ull * n);
  return s;
}

int64_t leaf_acc_chunk() {
  static int64_t v = -1;
  if (v < 0) {
    const char* e = getenv("NORTHUP_ACC_CHUNK");
    v = (e && atoll(e) >= 32) ? atoll(e) / 32 * 32 : kAccChunk;
  }
  return v;
}

static int sms_of(int dev) {
  static std::atomic<int> num_sms[kMaxDevices];
  if (num_sms[dev].load() == 0) {
    int n = 0;
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    num_sms[dev].store(n > 0 ? n : 148);
  }
  return num_sms[dev].load();
}

int leaf_run(const LeafCall& c) {
  using namespace leaf;
  const int64_t M = c.M, N = c.N, K = c.K;
  if (M < 0 || N < 0 || K < 0) return fail(NU_EINVAL, "negative dimension");
  if (M == 0 || N == 0) return 0;
  if (K == 0) {
    if (c.accumulate) return 0;
    cudaError_t e = cudaMemset2DAsync(c.C, c.ldc * 4, 0, N * 4, M, c.stream);
    return e == cudaSuccess ? 0 : fail(NU_ECUDA, "memset: %s", cudaGetErrorString(e));
  }
  if (M > INT32_MAX || N > INT32_MAX || K > INT32_MAX) return fail(NU_EINVAL, "dimension exceeds int32");
  if (c.lda < K || c.ldb < N || c.ldc < N) return fail(NU_EINVAL, "leading dimension too small");
  if (!c.A || !c.B || !c.C) return fail(NU_EINVAL, "null operand");
  if (c.eb_presplit && (c.ldb % 8 || reinterpret_cast<uintptr_t>(c.B) % 16))
    return fail(NU_EINVAL, "pre-split B needs a 16-B aligned base and ldb %% 8 == 0");
  if (!c.eb_presplit && N > split_b_max_n())
    return fail(NU_EINVAL, "leaf N = %lld above %lld", (long long)N, (long long)split_b_max_n());
  int64_t panel = c.panel > 0 ? c.panel : kDefaultKChunk;
  panel = (panel + 31) / 32 * 32;
  const int npass = (c.npass == 1 || c.npass == 4) ? c.npass : 3;
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= kMaxDevices) return fail(NU_EINVAL, "device ordinal out of range");
  const int sms = sms_of(dev);
  static int env_band = -1;
  if (env_band < 0) {
    const char* v = getenv("NORTHUP_RASTER_BAND");
    env_band = (v && atoi(v) > 0) ? atoi(v) : kRasterBand;
  }
  const int64_t pk = std::min<int64_t>(panel, (K + 31) / 32 * 32);
  const uint64_t need = leaf_scratch_bytes(M, N, pk, c.eb_presplit != nullptr);
  char* scratch = c.scratch;
  bool pooled = false;
  if (!scratch) {
    int rc = scratch_alloc(dev, need, c.stream, &scratch);
    if (rc) return rc;
    pooled = true;
  } else if (c.scratch_bytes < need) {
    return fail(NU_ENOMEM, "leaf scratch %llu B < %llu B", (unsigned long long)c.scratch_bytes,
                (unsigned long long)need);
  }
  const int64_t Kp = (pk + 31) / 32 * 32;
  float* Ap = reinterpret_cast<float*>(scratch);
  int* ea = reinterpret_cast<int*>(scratch + al256(4ull * M * Kp));
  char* bpart = scratch + al256(4ull * M * Kp) + al256(4ull * M);
  const int64_t ldq = (N + 31) / 32 * 32;
  float* Bp = reinterpret_cast<float*>(bpart);
  int* eb = reinterpret_cast<int*>(bpart + al256(4ull * Kp * ldq));
  unsigned* bmax = reinterpret_cast<unsigned*>(bpart + al256(4ull * Kp * ldq) + al256(4ull * N));
  const int64_t acc = std::min<int64_t>(leaf_acc_chunk(), Kp);
  int rc = 0;
  for (int64_t k0 = 0, p = 0; k0 < K && rc == 0; k0 += panel, ++p) {
    const int kl = static_cast<int>(std::min(panel, K - k0));
    rc = split_a_launch(c.A + k0, c.lda, static_cast<int>(M), kl, Ap, Kp, ea, sms, c.stream);
    SplitOperand sa{Ap, Kp, ea}, sb{};
    if (rc == 0) {
      if (c.eb_presplit) {
        sb = SplitOperand{c.B + k0 * c.ldb, c.ldb, c.eb_presplit + p * c.eb_stride};
      } else {
        rc = split_b_launch(c.B + k0 * c.ldb, c.ldb, kl, static_cast<int>(N), Bp, ldq, eb, bmax, c.stream);
        sb = SplitOperand{Bp, ldq, eb};
      }
    }
    if (rc == 0)
      rc = x3_gemm(sa, sb, c.C, c.ldc, static_cast<int>(M), static_cast<int>(N), kl,
                   (k0 > 0 || c.accumulate) ? 1 : 0, static_cast<int>((acc + 31) / 32), npass, env_band, sms, dev,
                   c.dbg, c.stream);
  }
  if (pooled) cudaFreeAsync(scratch, c.stream);
  return rc;
}

// variant: 0 = default (env NORTHUP_LEAF=1..5 may override), 1 = v0 (1 CTA), 2 = v1.2 (pair),
// 3 = v2 (pair, LDG-fed), 4 = v3 (pair, A' in TMEM).
int leaf_gemm_launch_dbg(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                         int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t kc,
                         int npass, int b_kmajor, float* dbg, int variant, cudaStream_t stream) {
  using namespace leaf;
  if (variant == 0) variant = default_leaf_variant();
  if (variant == 5) {
    if (b_kmajor) return fail(NU_EINVAL, "the leaf takes B row-major (K x N)");
    LeafCall c{};
    c.A = A, c.lda = lda, c.B = B, c.ldb = ldb, c.C = C, c.ldc = ldc, c.M = M, c.N = N, c.K = K;
    c.accumulate = accumulate, c.panel = kc, c.npass = npass, c.dbg = dbg, c.stream = stream;
    return leaf_run(c);
  }
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
