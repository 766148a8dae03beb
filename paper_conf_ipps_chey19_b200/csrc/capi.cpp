// C ABI entry points for the GEMM, the leaf, plan introspection and the
// partitioner (include/northup.h).
#include <errno.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <vector>

#include <chrono>

#include "northup_internal.h"

using namespace nu;


static double now_ms() {
  using namespace std::chrono;
  return duration<double, std::milli>(steady_clock::now().time_since_epoch()).count();
}

extern "C" {

int northup_leaf_gemm(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                      int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t k_chunk,
                      int npass, void* stream) {
  if ((!A || !B) && M > 0 && N > 0 && K > 0) return fail(NU_EINVAL, "NULL operand");
  if (!C && M > 0 && N > 0) return fail(NU_EINVAL, "NULL C");
  return leaf_gemm_launch(A, lda, B, ldb, C, ldc, M, N, K, accumulate,
                          k_chunk > 0 ? k_chunk : kDefaultKChunk, npass, static_cast<cudaStream_t>(stream));
}

int northup_gemm(northup_tree_t t, northup_buf_t A, northup_buf_t B, northup_buf_t C, int64_t M,
                 int64_t N, int64_t K) {
  return northup_gemm_ex(t, A, B, C, M, N, K, nullptr, nullptr);
}

static int zero_root_c(northup_tree_t t, northup_buf_t C, int64_t M, int64_t N) {
  const uint64_t bytes = static_cast<uint64_t>(M) * N * 4;
  if (C->storage == NU_HOST) {
    memset(C->ptr, 0, bytes);
    return 0;
  }
  if (C->storage == NU_HBM) {
    cudaSetDevice(t->nodes[C->node].phys);
    cudaError_t e = cudaMemset(C->ptr, 0, bytes);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    return e == cudaSuccess ? 0 : cuda_fail(e, "cudaMemset");
  }
  return fail(NU_ENOTSUP, "K == 0 on a FILE root");
}

int northup_gemm_ex(northup_tree_t t, northup_buf_t A, northup_buf_t B, northup_buf_t C, int64_t M,
                    int64_t N, int64_t K, const northup_gemm_opts* o, northup_stats* s) {
  const double t0 = now_ms();
  if (!t || !A || !B || !C) return fail(NU_EINVAL, "NULL argument");
  if (!t->finalized) return fail(NU_ESTATE, "tree not finalized");
  if (t->busy) return fail(NU_ESTATE, "a northup_gemm is already in flight on this tree");
  if (M < 0 || N < 0 || K < 0) return fail(NU_EINVAL, "negative dimension");
  if (A->tree != t || B->tree != t || C->tree != t) return fail(NU_EINVAL, "buffer from another tree");
  if (A->node != 0 || B->node != 0 || C->node != 0)
    return fail(NU_EINVAL, "A, B and C must live at the root node (level 0)");
  // multi-process siblings pass only their own strips (northup_tree_set_local)
  int64_t m = M, n = N;
  if (t->local_node >= 0) {
    const auto& ch = t->nodes[0].children;
    const int G = static_cast<int>(ch.size());
    const int idx = static_cast<int>(std::find(ch.begin(), ch.end(), t->local_node) - ch.begin());
    int64_t r0, r1, c0, c1;
    int rc = region_of(G, M, N, idx, &r0, &r1, &c0, &c1);
    if (rc) return rc;
    m = r1 - r0;
    n = c1 - c0;
  }
  const uint64_t need_a = 4ull * m * K, need_b = 4ull * K * n, need_c = 4ull * m * n;
  if (A->bytes < need_a || B->bytes < need_b || C->bytes < need_c)
    return fail(NU_EINVAL, "buffer smaller than its matrix");
  if (o && o->replicate_result && t->nodes[0].storage == NU_FILE)
    return fail(NU_ENOTSUP, "replicate_result from a FILE root is not supported");
  northup_stats local{};
  northup_stats* st = s ? s : &local;
  *st = northup_stats{};
  if (M == 0 || N == 0) return 0;
  if (K == 0) return zero_root_c(t, C, m, n);
  if (t->nodes[0].storage == NU_FILE &&
      (A->storage != NU_FILE || B->storage != NU_FILE || C->storage != NU_FILE))
    return fail(NU_EINVAL, "a FILE root needs A, B and C as files (northup_open_file / alloc)");

  if (o && o->schedule == NU_SCHED_QUEUE && (t->nodes[0].storage != NU_HOST || t->local_node >= 0))
    return fail(NU_ENOTSUP, "NU_SCHED_QUEUE needs a HOST root in one process");
  t->busy = true;
  Plan plan;
  const bool a_al = reinterpret_cast<uintptr_t>(A->ptr) % 16 == 0;
  const bool b_al = reinterpret_cast<uintptr_t>(B->ptr) % 16 == 0;
  int rc = build_plan_ex(t, M, N, K, o, a_al, b_al, &plan);
  const double t1 = now_ms();
  if (!rc) {
    *st = plan.stats;
    st->t_plan_ms = t1 - t0;
    int prev = 0;
    cudaGetDevice(&prev);
    if (o && o->schedule == NU_SCHED_QUEUE)
      rc = execute_queue(t, M, N, K, A, B, C, o, st);   // tiles popped at run time
    else
      rc = execute_plan(t, plan, A, B, C, o, st);
    // replicas: pushed by the plan's own copies, else gathered after the join
    if (!rc && o && o->replicate_result && !plan.replica_push) rc = gather_replicas(t, plan, C, st);
    cudaSetDevice(prev);
  }
  t->busy = false;
  st->t_total_ms = now_ms() - t0;
  return rc;
}

// ------------------------------------------------------------ plan API
int northup_plan_create(northup_tree_t t, int64_t M, int64_t N, int64_t K,
                        const northup_gemm_opts* opts, northup_plan_t* out) {
  if (!t || !out) return fail(NU_EINVAL, "NULL argument");
  northup_plan_s* p = new northup_plan_s();
  int rc = build_plan(t, M, N, K, opts, &p->plan);
  if (rc) {
    delete p;
    return rc;
  }
  *out = p;
  return 0;
}

int northup_plan_num_ops(northup_plan_t p, int64_t* n) {
  if (!p || !n) return fail(NU_EINVAL, "NULL argument");
  *n = static_cast<int64_t>(p->plan.ops.size());
  return 0;
}

int northup_plan_get_op(northup_plan_t p, int64_t i, northup_op* out) {
  if (!p || !out || i < 0 || i >= static_cast<int64_t>(p->plan.ops.size()))
    return fail(NU_EINVAL, "bad op index");
  *out = p->plan.ops[i];
  return 0;
}

int northup_plan_num_bufs(northup_plan_t p, int* n) {
  if (!p || !n) return fail(NU_EINVAL, "NULL argument");
  *n = static_cast<int>(p->plan.bufs.size());
  return 0;
}

int northup_plan_get_buf(northup_plan_t p, int i, northup_plan_buf* out) {
  if (!p || !out || i < 0 || i >= static_cast<int>(p->plan.bufs.size()))
    return fail(NU_EINVAL, "bad buffer index");
  const PlanBuf& b = p->plan.bufs[i];
  out->kind = b.kind;
  out->node = b.node;
  out->worker = b.worker;
  out->bytes = b.bytes;
  return 0;
}

int northup_plan_stats(northup_plan_t p, northup_stats* out) {
  if (!p || !out) return fail(NU_EINVAL, "NULL argument");
  *out = p->plan.stats;
  return 0;
}

int northup_plan_destroy(northup_plan_t p) {
  delete p;
  return 0;
}

// ------------------------------------------- file preprocessing (R15)
int northup_file_tile_kpanels(const char* src, const char* dst, int64_t M, int64_t K,
                              int64_t panel_k) {
  if (!src || !dst || M < 0 || K < 0 || panel_k <= 0) return fail(NU_EINVAL, "bad arguments");
  FILE* in = fopen(src, "rb");
  if (!in) return fail(NU_EIO, "open %s: %s", src, strerror(errno));
  FILE* out = fopen(dst, "wb");
  if (!out) {
    fclose(in);
    return fail(NU_EIO, "open %s: %s", dst, strerror(errno));
  }
  // Stream row blocks of A; scatter each row's panel pieces to their panels.
  const int64_t rows_per = std::max<int64_t>(1, (256ll << 20) / std::max<int64_t>(1, K * 4));
  std::vector<float> buf(static_cast<size_t>(rows_per * K));
  int rc = 0;
  for (int64_t r0 = 0; r0 < M && !rc; r0 += rows_per) {
    const int64_t nr = std::min(rows_per, M - r0);
    if (fread(buf.data(), 4, static_cast<size_t>(nr * K), in) != static_cast<size_t>(nr * K)) {
      rc = fail(NU_EIO, "short read from %s", src);
      break;
    }
    for (int64_t k0 = 0; k0 < K && !rc; k0 += panel_k) {
      const int64_t w = std::min(panel_k, K - k0);
      // panel p starts at element k0 * M; row r of the panel at + r * w
      if (fseeko(out, static_cast<off_t>((k0 * M + r0 * w) * 4), SEEK_SET) != 0) {
        rc = fail(NU_EIO, "seek %s: %s", dst, strerror(errno));
        break;
      }
      for (int64_t r = 0; r < nr; ++r)
        if (fwrite(buf.data() + r * K + k0, 4, static_cast<size_t>(w), out) != static_cast<size_t>(w)) {
          rc = fail(NU_EIO, "write %s: %s", dst, strerror(errno));
          break;
        }
    }
  }
  fclose(in);
  if (fclose(out) != 0 && !rc) rc = fail(NU_EIO, "close %s: %s", dst, strerror(errno));
  return rc;
}

// --------------------------------------------------------- partitioner
int northup_partition(int G, int64_t M, int64_t N, int64_t K, int* Pr, int* Pc) {
  (void)K;
  if (!Pr || !Pc) return fail(NU_EINVAL, "NULL argument");
  return partition_grid(G, M, N, Pr, Pc);
}

int northup_partition_region(int G, int64_t M, int64_t N, int64_t K, int r, int64_t* r0,
                             int64_t* r1, int64_t* c0, int64_t* c1) {
  (void)K;
  if (!r0 || !r1 || !c0 || !c1) return fail(NU_EINVAL, "NULL argument");
  return region_of(G, M, N, r, r0, r1, c0, c1);
}

}  // extern "C"
