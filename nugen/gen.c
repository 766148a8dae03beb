/*
 * nugen — seeded, counter-based synthetic input generator shared by the CUDA
 * path's harness (bench.py, tests) and by the oracle's checks.
 *
 * It holds NONE of the method's arithmetic (no products, sums or blocking):
 * it only maps a global coordinate (i, j) of matrix `mat` to a value, so any
 * sub-block of a matrix can be regenerated independently and in parallel.
 * The recipe is SURVEY.md §8(d) "Concrete synthetic inputs":
 *
 *   h(seed, mat, i, j) = splitmix64((seed * 0x9E3779B97F4A7C15)
 *                                   ^ (mat << 56) ^ (i * ncols + j))
 *   uniform : ((h >> 40) - 2^23) * 2^-23          in [-1, 1), exact fp32
 *   int     : (h mod 17) - 8                      in [-8, 8]
 *   eye     : 1 if i == j else 0
 *   ones    : 1
 *   rank1   : u(i) * v(j), u(i) = (h(seed,mat,i,0x0F0F..)&7)-3,
 *                          v(j) = (h(seed,mat^0x40,j,0x0F0F..)&7)-3  (small ints)
 *   zeros   : 0
 *   temp    : (float)(330 + 10 u)   HotSpot-2D temperature grid, K   (u = uniform)
 *   power   : (float)(0.25 + 0.25 u) HotSpot-2D power grid, in [0, 0.5) (exact fp32)
 *
 * The paper's workload is "16k x 16k and 32k x 32k float matrices" (PAPER.md
 * P:349, §V-A); values are unspecified there, so the distribution is ours.
 */
#include <stdint.h>
#include <stddef.h>

#define NUGEN_UNIFORM 0
#define NUGEN_INT 1
#define NUGEN_EYE 2
#define NUGEN_ONES 3
#define NUGEN_RANK1 4
#define NUGEN_ZEROS 5
#define NUGEN_TEMP 6
#define NUGEN_POWER 7

static inline uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

static inline uint64_t nugen_hash(uint64_t seed, uint64_t mat, uint64_t idx) {
  return splitmix64((seed * 0x9E3779B97F4A7C15ULL) ^ (mat << 56) ^ idx);
}

static inline float nugen_value(int kind, uint64_t seed, uint64_t mat,
                                int64_t ncols, int64_t i, int64_t j) {
  switch (kind) {
    case NUGEN_UNIFORM: {
      uint64_t h = nugen_hash(seed, mat, (uint64_t)i * (uint64_t)ncols + (uint64_t)j);
      int64_t q = (int64_t)(h >> 40) - (1LL << 23);
      return (float)q * (1.0f / 8388608.0f);
    }
    case NUGEN_TEMP:
    case NUGEN_POWER: {
      uint64_t h = nugen_hash(seed, mat, (uint64_t)i * (uint64_t)ncols + (uint64_t)j);
      double u = (double)((int64_t)(h >> 40) - (1LL << 23)) * (1.0 / 8388608.0);
      return kind == NUGEN_TEMP ? (float)(330.0 + 10.0 * u) : (float)(0.25 + 0.25 * u);
    }
    case NUGEN_INT: {
      uint64_t h = nugen_hash(seed, mat, (uint64_t)i * (uint64_t)ncols + (uint64_t)j);
      return (float)((int64_t)(h % 17ULL) - 8);
    }
    case NUGEN_EYE:
      return i == j ? 1.0f : 0.0f;
    case NUGEN_ONES:
      return 1.0f;
    case NUGEN_RANK1: {
      uint64_t hu = nugen_hash(seed, mat, (uint64_t)i ^ 0x0F0F0F0F0F0FULL);
      uint64_t hv = nugen_hash(seed, mat ^ 0x40ULL, (uint64_t)j ^ 0x0F0F0F0F0F0FULL);
      return (float)(((int64_t)(hu & 7ULL) - 3) * ((int64_t)(hv & 7ULL) - 3));
    }
    default:
      return 0.0f;
  }
}

/* Fill the rows x cols sub-block whose top-left global coordinate is (i0, j0)
 * of a matrix with `ncols` columns; out is row-major with leading dim ld. */
void nugen_fill_f32(float* out, int64_t ld, uint64_t seed, int mat, int kind,
                    int64_t ncols, int64_t i0, int64_t j0, int64_t rows,
                    int64_t cols) {
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < rows; ++r) {
    float* o = out + r * ld;
    for (int64_t c = 0; c < cols; ++c)
      o[c] = nugen_value(kind, seed, (uint64_t)mat, ncols, i0 + r, j0 + c);
  }
}

/* Scalar accessor, for spot checks. */
float nugen_entry(uint64_t seed, int mat, int kind, int64_t ncols, int64_t i,
                  int64_t j) {
  return nugen_value(kind, seed, (uint64_t)mat, ncols, i, j);
}
