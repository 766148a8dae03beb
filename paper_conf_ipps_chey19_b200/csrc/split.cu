// Operand split of the leaf (R22): every fp32 operand x of one K
// panel is written as
//
//     x = 2^e (hi + lo),   hi = fp16_rn(x 2^-e),   lo = fp16_rn(x 2^-e - hi)
//
// with one power-of-two exponent e per ROW of A and per COLUMN of B (over the
// panel's K range), chosen so that the row's (column's) largest |x| 2^-e lies
// in [2^14, 2^15): every hi is a normal fp16 (11 significant bits, so any
// fp16 x fp16 tensor-core product is exact) for elements down to 2^-28 of the
// row maximum, and x 2^-e - hi is exact in fp32.  The leaf computes
// hi_a hi_b + hi_a lo_b + lo_a hi_b with three fp16 MMAs per 16 k and scales
// the accumulator by 2^(e_i + e_j) (exact).  Error per product
// <= 3 * 2^-22 |a||b| (R22), against the 1e-5 normwise bound of BJ.
//
// The split is the fp32 -> fp16 conversion on the HBM -> SMEM edge:
// it runs once per K panel, and the split operand has exactly the bytes of
// the fp32 panel (two fp16 per element), so the GEMM's TMA moves what the raw
// panel would and the split may run in place.
//
// Layouts (ld = the fp32 row stride of the buffer, in floats):
//   A' row i at byte 4 ld i; 32-k stage s occupies the stage's own 128 bytes:
//      fp16 [64 s + (k % 32)] = hi, [64 s + 32 + (k % 32)] = lo
//   B' row k at byte 4 ld k: fp16 [n] = hi, [ld + n] = lo
// Panels are zero-padded to Kp = K rounded up to 32 (rows / columns [K, Kp)
// must exist in the destination).
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "leaf_common.cuh"
#include "northup_internal.h"

namespace nu {
namespace leaf {

// e with amax 2^-e in [2^14, 2^15), clamped so that 2^-e is a normal float
// (rows of zeros, or maxima outside [2^-112, 2^127), are not normalised).
__device__ __forceinline__ int split_exponent(float amax) {
  int E = static_cast<int>((__float_as_uint(amax) >> 23) & 0xFF);
  if (E == 0) E = 1;
  const int e = E - 141;
  return e < -126 ? -126 : (e > 126 ? 126 : e);
}

__device__ __forceinline__ float pow2(int e) {   // e in [-126, 127]
  return __uint_as_float(static_cast<uint32_t>(e + 127) << 23);
}

__device__ __forceinline__ void split1(float x, float s, __half& hi, __half& lo) {
  const float y = x * s;                        // exact: s is a power of two
  hi = __float2half_rn(y);
  lo = __float2half_rn(y - __half2float(hi));   // y - hi is exact in fp32
}

// hi / lo of four consecutive k (or n) as two 8-byte stores' worth of fp16
__device__ __forceinline__ void split4(float4 x, float s, uint2& hi, uint2& lo) {
  __half h[4], l[4];
  split1(x.x, s, h[0], l[0]);
  split1(x.y, s, h[1], l[1]);
  split1(x.z, s, h[2], l[2]);
  split1(x.w, s, h[3], l[3]);
  hi = make_uint2(__half_as_ushort(h[0]) | (static_cast<uint32_t>(__half_as_ushort(h[1])) << 16),
                  __half_as_ushort(h[2]) | (static_cast<uint32_t>(__half_as_ushort(h[3])) << 16));
  lo = make_uint2(__half_as_ushort(l[0]) | (static_cast<uint32_t>(__half_as_ushort(l[1])) << 16),
                  __half_as_ushort(l[2]) | (static_cast<uint32_t>(__half_as_ushort(l[3])) << 16));
}

// One warp per row of A (grid-stride).  Pass 1: row max; pass 2: each 32-k
// group is read by the warp, then written (the same 128 bytes when in place).
// vec: A and dst rows 16-B aligned (float4 loads, 128 k per warp step).
__device__ __forceinline__ void split_a_rows(const float* A, int64_t lda, int M, int Kl, int Kp, float* dst,
                                             int64_t ldd, int* ea, int vec, int block, int blocks) {
  const int lane = threadIdx.x & 31;
  const int warps = (blocks * blockDim.x) >> 5;
  for (int r = (block * blockDim.x + threadIdx.x) >> 5; r < M; r += warps) {
    const float* a = A + static_cast<int64_t>(r) * lda;
    float m = 0.f;
    if (vec) {
      const int K4 = Kl & ~3;
      for (int k = 4 * lane; k < K4; k += 128) {
        const float4 x = *reinterpret_cast<const float4*>(a + k);
        m = fmaxf(fmaxf(m, fmaxf(fabsf(x.x), fabsf(x.y))), fmaxf(fabsf(x.z), fabsf(x.w)));
      }
      for (int k = K4 + lane; k < Kl; k += 32) m = fmaxf(m, fabsf(a[k]));
    } else {
      for (int k = lane; k < Kl; k += 32) m = fmaxf(m, fabsf(a[k]));
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    const int e = split_exponent(m);
    if (lane == 0) ea[r] = e;
    const float s = pow2(-e);
    __half* out = reinterpret_cast<__half*>(dst + static_cast<int64_t>(r) * ldd);
    int kv = 0;
    if (vec) {
      // lane l: k = k0 + 4 l .. +3, i.e. group g = l / 8, positions 4 (l % 8) .. +3
      for (; kv + 128 <= Kl; kv += 128) {
        const float4 x = *reinterpret_cast<const float4*>(a + kv + 4 * lane);
        __syncwarp();                            // the 512 bytes are read before they are overwritten
        uint2 hi, lo;
        split4(x, s, hi, lo);
        const int g = lane >> 3, c = 4 * (lane & 7);
        *reinterpret_cast<uint2*>(out + 2 * (kv + 32 * g) + c) = hi;
        *reinterpret_cast<uint2*>(out + 2 * (kv + 32 * g) + 32 + c) = lo;
        __syncwarp();
      }
    }
    for (int k0 = kv; k0 < Kp; k0 += 32) {
      const int k = k0 + lane;
      const float x = k < Kl ? a[k] : 0.f;
      __syncwarp();                              // the group is read before it is overwritten
      __half hi, lo;
      split1(x, s, hi, lo);
      out[2 * k0 + lane] = hi;
      out[2 * k0 + 32 + lane] = lo;
      __syncwarp();
    }
  }
}

__global__ void __launch_bounds__(256) split_a_kernel(const float* A, int64_t lda, int M, int Kl, int Kp,
                                                      float* dst, int64_t ldd, int* ea, int vec) {
  split_a_rows(A, lda, M, Kl, Kp, dst, ldd, ea, vec, blockIdx.x, gridDim.x);
}

// Few rows (a 1024-row strip of S2B's second phase): four warps per row, each
// over a quarter of the panel's K (a multiple of 32 k, so no 32-k group is
// shared), the row maximum combined through shared memory.  The same exponent
// and the same per-element conversion as split_a_rows: bitwise the same split,
// with four times the warps in flight (a warp per row left ~7 per SM).
__global__ void __launch_bounds__(256) split_a_quarters_kernel(const float* A, int64_t lda, int M, int Kl, int Kp,
                                                               int Q, float* dst, int64_t ldd, int* ea, int vec) {
  __shared__ float mx[2][4];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int r = blockIdx.x * 2 + (warp >> 2), q = warp & 3;
  const int k0 = q * Q, k1 = min(Kp, k0 + Q), kl1 = min(Kl, k1);
  const float* a = A + static_cast<int64_t>(min(r, M - 1)) * lda;
  float m = 0.f;
  if (r < M) {
    int k = k0;
    if (vec)
      for (; k + 128 <= kl1; k += 128) {
        const float4 x = *reinterpret_cast<const float4*>(a + k + 4 * lane);
        m = fmaxf(fmaxf(m, fmaxf(fabsf(x.x), fabsf(x.y))), fmaxf(fabsf(x.z), fabsf(x.w)));
      }
    for (k += lane; k < kl1; k += 32) m = fmaxf(m, fabsf(a[k]));
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  if (lane == 0) mx[warp >> 2][q] = m;
  __syncthreads();
  if (r >= M) return;
  const float* mr = mx[warp >> 2];
  const int e = split_exponent(fmaxf(fmaxf(mr[0], mr[1]), fmaxf(mr[2], mr[3])));
  if (q == 0 && lane == 0) ea[r] = e;
  const float s = pow2(-e);
  __half* out = reinterpret_cast<__half*>(dst + static_cast<int64_t>(r) * ldd);
  int kv = k0;
  if (vec) {
    for (; kv + 128 <= kl1; kv += 128) {
      const float4 x = *reinterpret_cast<const float4*>(a + kv + 4 * lane);
      __syncwarp();                            // the 512 bytes are read before they are overwritten
      uint2 hi, lo;
      split4(x, s, hi, lo);
      const int g = lane >> 3, c = 4 * (lane & 7);
      *reinterpret_cast<uint2*>(out + 2 * (kv + 32 * g) + c) = hi;
      *reinterpret_cast<uint2*>(out + 2 * (kv + 32 * g) + 32 + c) = lo;
      __syncwarp();
    }
  }
  for (int g0 = kv; g0 < k1; g0 += 32) {
    const int k = g0 + lane;
    const float x = k < Kl ? a[k] : 0.f;
    __syncwarp();                              // the group is read before it is overwritten
    __half hi, lo;
    split1(x, s, hi, lo);
    out[2 * g0 + lane] = hi;
    out[2 * g0 + 32 + lane] = lo;
    __syncwarp();
  }
}

// Small panels (cfg1-like leaf calls): the A split and the whole B split
// (column maxima, exponents, hi / lo) in ONE launch instead of five.  Blocks
// [0, ga) split rows of A as split_a_kernel does; each further block takes 32
// columns of B: lane = column, the 8 warps stride over the panel's rows, a
// shared-memory max per column, then the split (out of place).
__global__ void __launch_bounds__(256) split_ab_small_kernel(const float* A, int64_t lda, int M, int Kl, int Kp,
                                                             float* adst, int64_t ldda, int* ea, int avec, int ga,
                                                             const float* B, int64_t ldb, int N, float* bdst,
                                                             int64_t lddb, int* eb) {
  if (static_cast<int>(blockIdx.x) < ga) {
    split_a_rows(A, lda, M, Kl, Kp, adst, ldda, ea, avec, blockIdx.x, ga);
    return;
  }
  __shared__ float cmax[8][32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int n = (blockIdx.x - ga) * 32 + lane;
  float m = 0.f;
  if (n < N)
    for (int k = warp; k < Kl; k += 8) m = fmaxf(m, fabsf(B[static_cast<int64_t>(k) * ldb + n]));
  cmax[warp][lane] = m;
  __syncthreads();
  if (warp == 0) {
#pragma unroll
    for (int w = 1; w < 8; ++w) m = fmaxf(m, cmax[w][lane]);
    cmax[0][lane] = m;
  }
  __syncthreads();
  if (n >= N) return;
  const int e = split_exponent(cmax[0][lane]);
  if (warp == 0) eb[n] = e;
  const float sc = pow2(-e);
  for (int k = warp; k < Kp; k += 8) {
    __half h, l;
    split1(k < Kl ? B[static_cast<int64_t>(k) * ldb + n] : 0.f, sc, h, l);
    __half* hi_row = reinterpret_cast<__half*>(bdst + static_cast<int64_t>(k) * lddb);
    hi_row[n] = h;
    hi_row[lddb + n] = l;
  }
}

// Column maxima of B (|x| as uint bits; atomicMax over 256-row slabs).
__global__ void __launch_bounds__(256) colmax_kernel(const float* B, int64_t ldb, int Kl, int N,
                                                     unsigned* bmax) {
  const int n = blockIdx.x * 256 + threadIdx.x;
  if (n >= N) return;
  const int k0 = blockIdx.y * 256, k1 = min(Kl, k0 + 256);
  float m = 0.f;
  for (int k = k0; k < k1; ++k) m = fmaxf(m, fabsf(B[static_cast<int64_t>(k) * ldb + n]));
  atomicMax(bmax + n, __float_as_uint(m));
}

// Column exponents from the column maxima (once per column, not per element).
__global__ void __launch_bounds__(256) col_exps_kernel(const unsigned* bmax, int N, int* eb) {
  const int n = blockIdx.x * 256 + threadIdx.x;
  if (n < N) eb[n] = split_exponent(__uint_as_float(bmax[n]));
}

// Out of place: rows [k0, k0 + 8) x 4 columns per thread, float4 loads and
// 8-byte hi / lo stores (B and dst rows 16-B aligned, N % 4 == 0).
__global__ void __launch_bounds__(256) split_b_oop_kernel(const float* __restrict__ B, int64_t ldb, int Kl, int Kp,
                                                          int N, const int* __restrict__ eb,
                                                          float* __restrict__ dst, int64_t ldd) {
  const int n = 4 * (blockIdx.x * 256 + threadIdx.x);
  if (n >= N) return;
  const float s0 = pow2(-eb[n]), s1 = pow2(-eb[n + 1]), s2 = pow2(-eb[n + 2]), s3 = pow2(-eb[n + 3]);
  const int k1 = min(Kp, 8 * (blockIdx.y + 1));
  for (int k = 8 * blockIdx.y; k < k1; ++k) {
    float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
    if (k < Kl) x = *reinterpret_cast<const float4*>(B + static_cast<int64_t>(k) * ldb + n);
    __half h[4], l[4];
    split1(x.x, s0, h[0], l[0]);
    split1(x.y, s1, h[1], l[1]);
    split1(x.z, s2, h[2], l[2]);
    split1(x.w, s3, h[3], l[3]);
    __half* hi_row = reinterpret_cast<__half*>(dst + static_cast<int64_t>(k) * ldd);
    const int64_t lo_off = ldd;
    *reinterpret_cast<uint2*>(hi_row + n) =
        make_uint2(__half_as_ushort(h[0]) | (static_cast<uint32_t>(__half_as_ushort(h[1])) << 16),
                   __half_as_ushort(h[2]) | (static_cast<uint32_t>(__half_as_ushort(h[3])) << 16));
    *reinterpret_cast<uint2*>(hi_row + lo_off + n) =
        make_uint2(__half_as_ushort(l[0]) | (static_cast<uint32_t>(__half_as_ushort(l[1])) << 16),
                   __half_as_ushort(l[2]) | (static_cast<uint32_t>(__half_as_ushort(l[3])) << 16));
  }
}

// One CTA per row of B: the row is staged in shared memory before any of it
// is overwritten (in place, hi lands on the row's first half and lo on its
// second).  Rows [Kl, Kp) are written as zeros.
constexpr int kSplitRowMaxN = 49152;   // 192 KiB of fp32 staging
__global__ void __launch_bounds__(1024) split_b_kernel(const float* B, int64_t ldb, int Kl, int N,
                                                       const int* eb, float* dst, int64_t ldd) {
  extern __shared__ float row[];
  const int k = blockIdx.x;
  const float* brow = B + static_cast<int64_t>(k) * ldb;
  for (int n = threadIdx.x; n < N; n += blockDim.x) row[n] = k < Kl ? brow[n] : 0.f;
  __syncthreads();
  __half* hi_row = reinterpret_cast<__half*>(dst + static_cast<int64_t>(k) * ldd);
  __half* lo_row = hi_row + ldd;
  for (int n = threadIdx.x; n < N; n += blockDim.x) {
    __half h, l;
    split1(row[n], pow2(-eb[n]), h, l);
    hi_row[n] = h;
    lo_row[n] = l;
  }
}

// In place, vectorised (N % 4 == 0, 16-B aligned rows): one CTA of 1024
// threads per row holds the whole row in registers (float4 loads, at most 12
// per thread for N <= 49152), then writes the hi and lo halves as 8-byte
// stores.  The shared-memory version above (scalar 2-byte stores) moved a
// 32768-wide panel at ~1.5 TB/s.
constexpr int kSplitVecPerThread = 12;
__global__ void __launch_bounds__(1024) split_b_inplace_vec_kernel(float* B, int64_t ldb, int Kl, int N,
                                                                   const int* __restrict__ eb) {
  const int k = blockIdx.x;
  const int N4 = N / 4;
  float4* row = reinterpret_cast<float4*>(B + static_cast<int64_t>(k) * ldb);
  float4 x[kSplitVecPerThread];
#pragma unroll
  for (int j = 0; j < kSplitVecPerThread; ++j) {
    const int i = threadIdx.x + j * 1024;
    x[j] = (k < Kl && i < N4) ? row[i] : make_float4(0.f, 0.f, 0.f, 0.f);
  }
  __syncthreads();                                   // the whole row is read before any of it is overwritten
  __half* hi_row = reinterpret_cast<__half*>(row);
#pragma unroll
  for (int j = 0; j < kSplitVecPerThread; ++j) {
    const int i = threadIdx.x + j * 1024;
    if (i >= N4) break;
    const int n = 4 * i;
    __half h[4], l[4];
    split1(x[j].x, pow2(-eb[n]), h[0], l[0]);
    split1(x[j].y, pow2(-eb[n + 1]), h[1], l[1]);
    split1(x[j].z, pow2(-eb[n + 2]), h[2], l[2]);
    split1(x[j].w, pow2(-eb[n + 3]), h[3], l[3]);
    *reinterpret_cast<uint2*>(hi_row + n) =
        make_uint2(__half_as_ushort(h[0]) | (static_cast<uint32_t>(__half_as_ushort(h[1])) << 16),
                   __half_as_ushort(h[2]) | (static_cast<uint32_t>(__half_as_ushort(h[3])) << 16));
    *reinterpret_cast<uint2*>(hi_row + ldb + n) =
        make_uint2(__half_as_ushort(l[0]) | (static_cast<uint32_t>(__half_as_ushort(l[1])) << 16),
                   __half_as_ushort(l[2]) | (static_cast<uint32_t>(__half_as_ushort(l[3])) << 16));
  }
}

int64_t split_b_max_n() { return kSplitRowMaxN; }

int split_a_launch(const float* A, int64_t lda, int M, int Kl, float* dst, int64_t ldd, int* ea, int sms,
                   cudaStream_t s) {
  if (M <= 0) return 0;
  const int Kp = (Kl + 31) / 32 * 32;
  const int grid = static_cast<int>(std::min<int64_t>((M + 7) / 8, 32LL * sms));
  const int vec = (reinterpret_cast<uintptr_t>(A) % 16 == 0) && lda % 4 == 0 &&
                  (reinterpret_cast<uintptr_t>(dst) % 16 == 0) && ldd % 4 == 0;
  if (M < 8 * sms && Kp >= 4 * 128) {
    const int Q = (Kp / 4 + 127) / 128 * 128;   // a multiple of 128 k (the vector step) and of 32
    split_a_quarters_kernel<<<(M + 1) / 2, 256, 0, s>>>(A, lda, M, Kl, Kp, Q, dst, ldd, ea, vec);
  } else {
    split_a_kernel<<<grid, 256, 0, s>>>(A, lda, M, Kl, Kp, dst, ldd, ea, vec);
  }
  count_launches(1);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : fail(NU_ECUDA, "split_a launch: %s", cudaGetErrorString(e));
}

int split_b_launch(const float* B, int64_t ldb, int Kl, int N, float* dst, int64_t ldd, int* eb,
                   unsigned* bmax, cudaStream_t s) {
  if (N <= 0) return 0;
  if (N > split_b_max_n()) return fail(NU_EINVAL, "split_b: N = %d above %lld", N, (long long)split_b_max_n());
  const int Kp = (Kl + 31) / 32 * 32;
  cudaError_t e = cudaMemsetAsync(bmax, 0, sizeof(unsigned) * N, s);
  if (e != cudaSuccess) return fail(NU_ECUDA, "split_b memset: %s", cudaGetErrorString(e));
  if (Kl > 0) {
    colmax_kernel<<<dim3((N + 255) / 256, (Kl + 255) / 256), 256, 0, s>>>(B, ldb, Kl, N, bmax);
    count_launches(1);
  }
  col_exps_kernel<<<(N + 255) / 256, 256, 0, s>>>(bmax, N, eb);
  count_launches(1);
  const bool vec = dst != B && N % 4 == 0 && ldb % 4 == 0 && ldd % 4 == 0 &&
                   reinterpret_cast<uintptr_t>(B) % 16 == 0 && reinterpret_cast<uintptr_t>(dst) % 16 == 0;
  if (vec) {
    split_b_oop_kernel<<<dim3((N / 4 + 255) / 256, (Kp + 7) / 8), 256, 0, s>>>(B, ldb, Kl, Kp, N, eb, dst, ldd);
  } else if (dst == B && ldd == ldb && N % 4 == 0 && ldb % 4 == 0 && reinterpret_cast<uintptr_t>(B) % 16 == 0 &&
             N <= 4 * 1024 * kSplitVecPerThread) {
    split_b_inplace_vec_kernel<<<Kp, 1024, 0, s>>>(const_cast<float*>(B), ldb, Kl, N, eb);
  } else {
    static bool configured[kMaxDevices];
    int dev = 0;
    cudaGetDevice(&dev);
    if (!configured[dev]) {
      e = cudaFuncSetAttribute(split_b_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * kSplitRowMaxN);
      if (e != cudaSuccess) return fail(NU_ECUDA, "split_b attribute: %s", cudaGetErrorString(e));
      configured[dev] = true;
    }
    const int threads = std::min(1024, std::max(64, (N / 8 + 31) / 32 * 32));
    split_b_kernel<<<Kp, threads, 4 * static_cast<size_t>(N), s>>>(B, ldb, Kl, N, eb, dst, ldd);
  }
  count_launches(1);
  e = cudaGetLastError();
  return e == cudaSuccess ? 0 : fail(NU_ECUDA, "split_b launch: %s", cudaGetErrorString(e));
}

int split_ab_small_launch(const float* A, int64_t lda, int M, int Kl, float* adst, int64_t ldda, int* ea,
                          const float* B, int64_t ldb, int N, float* bdst, int64_t lddb, int* eb, cudaStream_t s) {
  const int Kp = (Kl + 31) / 32 * 32;
  const int ga = M > 0 ? (M + 7) / 8 : 0, gb = (N + 31) / 32;
  if (ga + gb == 0) return 0;
  const int avec = (reinterpret_cast<uintptr_t>(A) % 16 == 0) && lda % 4 == 0 &&
                   (reinterpret_cast<uintptr_t>(adst) % 16 == 0) && ldda % 4 == 0;
  split_ab_small_kernel<<<ga + gb, 256, 0, s>>>(A, lda, M, Kl, Kp, adst, ldda, ea, avec, ga, B, ldb, N, bdst, lddb,
                                                  eb);
  count_launches(1);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : fail(NU_ECUDA, "split_ab_small launch: %s", cudaGetErrorString(e));
}

void preload_split() {
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, split_a_kernel);
  cudaFuncGetAttributes(&fa, split_a_quarters_kernel);
  cudaFuncGetAttributes(&fa, colmax_kernel);
  cudaFuncGetAttributes(&fa, split_b_kernel);
  cudaFuncGetAttributes(&fa, split_b_oop_kernel);
  cudaFuncGetAttributes(&fa, split_b_inplace_vec_kernel);
  cudaFuncGetAttributes(&fa, col_exps_kernel);
  cudaFuncGetAttributes(&fa, split_ab_small_kernel);
}

}  // namespace leaf
}  // namespace nu
