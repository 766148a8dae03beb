// Host side of the leaf: TMA descriptor encoding, the leaf's scratch, and the
// per-K-panel sequence split -> GEMM (leaf_run).
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

}  // namespace leaf

static std::atomic<long long> g_launches{0};
void count_launches(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

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
  count_launches(1);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : cuda_fail(e, "flag_store_kernel");
}

// Load every kernel the executor may launch on the current device (see
// leaf_common.cuh preload_sm*): run before work that waits on other processes.
void preload_kernels() {
  leaf::preload_x3();
  hotspot_preload();
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, debug_spin_kernel);
  cudaFuncGetAttributes(&fa, flag_store_kernel);
}

int debug_spin(long long ns, cudaStream_t s) {
  debug_spin_kernel<<<1, 1, 0, s>>>(ns);
  count_launches(1);
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
  const uint64_t nb = static_cast<uint64_t>(std::min<int64_t>(n, kLeafMaxN));
  uint64_t s = al256(4ull * m * Kp) + al256(4ull * m);
  if (!b_presplit) s += al256(4ull * Kp * ((nb + 31) / 32 * 32)) + 2 * al256(4ull * nb);
  return s;
}

int64_t leaf_acc_chunk() { return kAccChunk; }

// Panels with at most this many elements of A and B together take the fused
// one-launch split (split_ab_small_kernel).
constexpr int64_t kSplitSmallElems = int64_t(1) << 21;

int sms_of(int dev) {
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
  int64_t panel = c.panel > 0 ? c.panel : kDefaultKChunk;
  panel = (panel + 31) / 32 * 32;
  if (c.npass != 0 && c.npass != 1 && c.npass != 3 && c.npass != 4)
    return fail(NU_EINVAL, "npass %d: 0/3 (product), 1 (hi.hi only) or 4 (+ lo.lo)", c.npass);
  const int npass = c.npass == 0 ? kDefaultNpass : c.npass;
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= kMaxDevices) return fail(NU_EINVAL, "device ordinal out of range");
  const int sms = sms_of(dev);
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
  // B is split (and multiplied) kLeafMaxN columns at a time; A' is reused
  const int64_t NB = std::min<int64_t>(N, kLeafMaxN);
  const int64_t ldq = (NB + 31) / 32 * 32;
  float* Bp = reinterpret_cast<float*>(bpart);
  int* eb = reinterpret_cast<int*>(bpart + al256(4ull * Kp * ldq));
  unsigned* bmax = reinterpret_cast<unsigned*>(bpart + al256(4ull * Kp * ldq) + al256(4ull * NB));
  const int64_t acc = std::min<int64_t>(leaf_acc_chunk(), Kp);
  int rc = 0;
  for (int64_t k0 = 0, p = 0; k0 < K && rc == 0; k0 += panel, ++p) {
    const int kl = static_cast<int>(std::min(panel, K - k0));
    // small panels (cfg1's 64 x 64 x 64 blocks): both splits in one launch
    const bool small = !c.eb_presplit && N <= NB && static_cast<int64_t>(kl) * (M + N) <= kSplitSmallElems;
    if (small)
      rc = split_ab_small_launch(c.A + k0, c.lda, static_cast<int>(M), kl, Ap, Kp, ea, c.B + k0 * c.ldb, c.ldb,
                                 static_cast<int>(N), Bp, ldq, eb, c.stream);
    else
      rc = split_a_launch(c.A + k0, c.lda, static_cast<int>(M), kl, Ap, Kp, ea, sms, c.stream);
    const SplitOperand sa{Ap, Kp, ea};
    for (int64_t n0 = 0; n0 < N && rc == 0; n0 += NB) {
      const int nn = static_cast<int>(std::min(NB, N - n0));
      SplitOperand sb{};
      if (small) {
        sb = SplitOperand{Bp, ldq, eb};
      } else if (c.eb_presplit) {
        // split layout: column n0's hi sits 2 n0 bytes into the row
        const char* row = reinterpret_cast<const char*>(c.B + k0 * c.ldb) + 2 * n0;
        sb = SplitOperand{reinterpret_cast<const float*>(row), c.ldb, c.eb_presplit + p * c.eb_stride + n0};
      } else {
        rc = split_b_launch(c.B + k0 * c.ldb + n0, c.ldb, kl, nn, Bp, ldq, eb, bmax, c.stream);
        sb = SplitOperand{Bp, ldq, eb};
      }
      const bool ev = c.events && c.events_used && *c.events_used + 2 <= c.n_events;
      if (rc == 0 && ev) cudaEventRecord(c.events[*c.events_used], c.stream);
      if (rc == 0)
        rc = x3_gemm(sa, sb, c.C + n0, c.ldc, static_cast<int>(M), nn, kl, (k0 > 0 || c.accumulate) ? 1 : 0,
                     static_cast<int>((acc + 31) / 32), npass, kRasterBand, sms, dev, c.dbg, c.stream);
      if (rc == 0 && ev) {
        cudaEventRecord(c.events[*c.events_used + 1], c.stream);
        *c.events_used += 2;
      }
    }
  }
  if (pooled) cudaFreeAsync(scratch, c.stream);
  return rc;
}

int leaf_gemm_launch(const float* A, int64_t lda, const float* B, int64_t ldb, float* C, int64_t ldc, int64_t M,
                     int64_t N, int64_t K, int accumulate, int64_t kc, int npass, cudaStream_t stream) {
  LeafCall c{};
  c.A = A, c.lda = lda, c.B = B, c.ldb = ldb, c.C = C, c.ldc = ldc, c.M = M, c.N = N, c.K = K;
  c.accumulate = accumulate, c.panel = kc, c.npass = npass, c.stream = stream;
  return leaf_run(c);
}

}  // namespace nu

extern "C" long long northup_debug_kernel_launches(void) { return nu::g_launches.load(); }

// Debug entry (not part of northup.h): the leaf with CUDA events recorded
// around each GEMM kernel on `stream` (events: n_events cudaEvent_t handles;
// returns the number recorded in *used) — the bench's dominant-kernel timing.
extern "C" int northup_debug_leaf_gemm_events(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                                              int64_t ldc, int64_t M, int64_t N, int64_t K, int64_t kc,
                                              void* stream, void** events, int n_events, int* used) {
  nu::LeafCall c{};
  c.A = A, c.lda = lda, c.B = B, c.ldb = ldb, c.C = C, c.ldc = ldc, c.M = M, c.N = N, c.K = K;
  c.panel = kc, c.stream = static_cast<cudaStream_t>(stream);
  c.events = reinterpret_cast<cudaEvent_t*>(events), c.n_events = n_events, c.events_used = used;
  if (used) *used = 0;
  return nu::leaf_run(c);
}

// Debug entry (not part of northup.h): the leaf with a profile-mode counter
// buffer `dbg` (4 floats per CTA pair: cycles, MMA waits on data, MMA waits on
// the epilogue, stages).  b_kmajor must be 0 and variant 0.
extern "C" int northup_debug_leaf_gemm(const float* A, int64_t lda, const float* B, int64_t ldb,
                                       float* C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                                       int accumulate, int64_t kc, int npass, int b_kmajor,
                                       float* dbg, int variant, void* stream) {
  if (b_kmajor || (variant != 0 && variant != 5)) return nu::fail(NU_EINVAL, "unknown leaf variant");
  nu::LeafCall c{};
  c.A = A, c.lda = lda, c.B = B, c.ldb = ldb, c.C = C, c.ldc = ldc, c.M = M, c.N = N, c.K = K;
  c.accumulate = accumulate, c.panel = kc, c.npass = npass, c.dbg = dbg, c.stream = static_cast<cudaStream_t>(stream);
  return nu::leaf_run(c);
}
