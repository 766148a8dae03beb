/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct fp64 CPU reference for the Northup dense
 * matrix-multiply case study (§IV-A).  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load this library.  It shares no code, header or constant with the CUDA
 * path (paper_conf_ipps_chey19_b200/) and never includes anything from it.
 *
 * What it computes is the plain definition ("C = AB"; P:349
 * "float matrices"):
 *
 *     C_ref[i][j] = sum_{k=0}^{K-1} (double)A[i][k] * (double)B[k][j]
 *
 * with row-major A (M x K, ld lda), B (K x N, ld ldb) — DESIGN.md reading R1.
 *
 * Pins (tests/test_oracle.py): brute force on tiny inputs (2x2, 2x3.3x2),
 * closed forms (A.I = A, I.B = B, ones.ones = K, rank-1, diagonal scaling),
 * bitwise agreement with numpy.matmul(float64) on integer inputs, Freivalds
 * detects a planted error, the normwise checker flags a planted 2e-5 error.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int oracle_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

void oracle_set_threads(int n) {
#ifdef _OPENMP
  if (n > 0) omp_set_num_threads(n);
#else
  (void)n;
#endif
}

/* O1: the plain triple loop, fp64, i-k-j order (streams rows of B);
 * OpenMP over rows of C.  C is overwritten (reading R3: no alpha/beta). */
void oracle_gemm(const float* A, int64_t lda, const float* B, int64_t ldb,
                 double* C, int64_t ldc, int64_t M, int64_t N, int64_t K) {
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t i = 0; i < M; ++i) {
    double* c = C + i * ldc;
    for (int64_t j = 0; j < N; ++j) c[j] = 0.0;
    for (int64_t k = 0; k < K; ++k) {
      const double a = (double)A[i * lda + k];
      const float* b = B + k * ldb;
      for (int64_t j = 0; j < N; ++j) c[j] += a * (double)b[j];
    }
  }
}

/* O1 restricted to selected rows: out[r][j] = C_ref[rows[r]][j]. */
void oracle_gemm_rows(const float* A, int64_t lda, const float* B, int64_t ldb,
                      const int64_t* rows, int64_t nrows, double* out,
                      int64_t ldo, int64_t N, int64_t K) {
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t r = 0; r < nrows; ++r) {
    const int64_t i = rows[r];
    double* c = out + r * ldo;
    for (int64_t j = 0; j < N; ++j) c[j] = 0.0;
    for (int64_t k = 0; k < K; ++k) {
      const double a = (double)A[i * lda + k];
      const float* b = B + k * ldb;
      for (int64_t j = 0; j < N; ++j) c[j] += a * (double)b[j];
    }
  }
}

/* Sampled entries: out[s] = sum_k A[I[s]][k] * B[k][J[s]] in fp64. */
void oracle_entries(const float* A, int64_t lda, const float* B, int64_t ldb,
                    int64_t K, const int64_t* I, const int64_t* J, int64_t n,
                    double* out) {
#pragma omp parallel for schedule(static)
  for (int64_t s = 0; s < n; ++s) {
    double acc = 0.0;
    const float* a = A + I[s] * lda;
    for (int64_t k = 0; k < K; ++k) acc += (double)a[k] * (double)B[k * ldb + J[s]];
    out[s] = acc;
  }
}

/* Euclidean norms of the rows of A (M x K) and of the columns of B (K x N),
 * the scale of the normwise criterion (reading R10). */
void oracle_row_norms(const float* A, int64_t lda, int64_t M, int64_t K, double* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < M; ++i) {
    double s = 0.0;
    for (int64_t k = 0; k < K; ++k) {
      const double a = (double)A[i * lda + k];
      s += a * a;
    }
    out[i] = sqrt(s);
  }
}

void oracle_col_norms(const float* B, int64_t ldb, int64_t K, int64_t N, double* out) {
  double* acc = (double*)calloc((size_t)(N > 0 ? N : 1), sizeof(double));
  for (int64_t k = 0; k < K; ++k) {
    const float* b = B + k * ldb;
    for (int64_t j = 0; j < N; ++j) acc[j] += (double)b[j] * (double)b[j];
  }
  for (int64_t j = 0; j < N; ++j) out[j] = sqrt(acc[j]);
  free(acc);
}

/* Normwise error of a candidate C (fp32) against C_ref (fp64):
 *   max_{i,j} |C[i][j] - C_ref[i][j]| / (||A[i,:]||_2 * ||B[:,j]||_2)
 * Entries whose norm product is 0 must match exactly (else +inf).
 * Also returns the location of the maximum. */
double oracle_normwise_err(const float* C, int64_t ldc, const double* R, int64_t ldr,
                           const double* rn, const double* cn, int64_t M, int64_t N,
                           int64_t* arg_i, int64_t* arg_j) {
  double worst = 0.0;
  int64_t wi = -1, wj = -1;
  for (int64_t i = 0; i < M; ++i) {
    for (int64_t j = 0; j < N; ++j) {
      const double d = fabs((double)C[i * ldc + j] - R[i * ldr + j]);
      const double s = rn[i] * cn[j];
      double e;
      if (s > 0.0)
        e = d / s;
      else
        e = (d == 0.0) ? 0.0 : INFINITY;
      if (e != e) e = INFINITY; /* NaN in C */
      if (wi < 0 || e > worst) {
        worst = e;
        wi = i;
        wj = j;
      }
    }
  }
  if (arg_i) *arg_i = wi;
  if (arg_j) *arg_j = wj;
  return worst;
}

/* Freivalds' check (large configs): for a vector r,
 *   x = C r  (fp64 sums of the candidate C)  and  y = A (B r)  (fp64),
 * and the per-row ratio |x_i - y_i| / (||A_i||_2 * sum_j ||B_:,j||_2 |r_j|)
 * must stay within the normwise bound (a necessary condition).  r is given
 * by the caller (seeded +-1 entries).  Returns the maximum ratio. */
double oracle_freivalds(const float* A, int64_t lda, const float* B, int64_t ldb,
                        const float* C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                        const double* r, const double* rn, const double* cn,
                        double* x_out, double* y_out) {
  double* br = (double*)calloc((size_t)(K > 0 ? K : 1), sizeof(double));
#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < K; ++k) {
    double s = 0.0;
    for (int64_t j = 0; j < N; ++j) s += (double)B[k * ldb + j] * r[j];
    br[k] = s;
  }
  double scale_c = 0.0;
  for (int64_t j = 0; j < N; ++j) scale_c += cn[j] * fabs(r[j]);
  double worst = 0.0;
#pragma omp parallel for schedule(static) reduction(max : worst)
  for (int64_t i = 0; i < M; ++i) {
    double x = 0.0, y = 0.0;
    for (int64_t j = 0; j < N; ++j) x += (double)C[i * ldc + j] * r[j];
    for (int64_t k = 0; k < K; ++k) y += (double)A[i * lda + k] * br[k];
    if (x_out) x_out[i] = x;
    if (y_out) y_out[i] = y;
    const double s = rn[i] * scale_c;
    double e = (s > 0.0) ? fabs(x - y) / s : (x == y ? 0.0 : INFINITY);
    if (e != e) e = INFINITY;
    if (e > worst) worst = e;
  }
  free(br);
  return worst;
}
