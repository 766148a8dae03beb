// Executor: runs a plan on the GPUs of the tree.
//
// One host worker thread per HBM sibling (branch parallelism, Fig. 2).
// Each worker owns CUDA streams for the edges of its subtree: H2D copies
// (data_down), the leaf kernel (compute_task), D2H copies (data_up) and D2D
// layout copies.  Ops are issued in plan order; each dependency on an op of
// another stream becomes a cudaStreamWaitEvent, so transfers of later
// chunks overlap the computation of earlier ones ("overlapping computation
// and communications (i.e. OpenCL/CUDA streams) at the leaf node").
#include <chrono>
#include <thread>

#include "northup_internal.h"

struct WorkerState {
  int node = -1;
  int device = -1;
  cudaStream_t streams[nu::S_NUM] = {};
  std::vector<cudaEvent_t> events;       // one per op (reused across calls)
  std::vector<cudaEvent_t> tev;          // timing events (2 per op, timing mode)
};

namespace nu {

int finalize_workers(northup_tree_s* t) {
  int ndev = northup_device_count();
  for (const Node& n : t->nodes) {
    if (n.storage != NU_HBM) continue;
    if (n.phys >= ndev)
      return fail(NU_ECUDA, "HBM node %d names device %d but %d CUDA device(s) are visible", n.id,
                  n.phys, ndev);
    WorkerState* w = new WorkerState();
    w->node = n.id;
    w->device = n.phys;
    cudaError_t e = cudaSetDevice(n.phys);
    for (int s = 0; s < S_NUM && e == cudaSuccess; ++s)
      e = cudaStreamCreateWithFlags(&w->streams[s], cudaStreamNonBlocking);
    t->workers.push_back(w);
    if (e != cudaSuccess) return cuda_fail(e, "stream creation");
  }
  return 0;
}

void destroy_workers(northup_tree_s* t) {
  for (WorkerState* w : t->workers) {
    cudaSetDevice(w->device);
    for (cudaStream_t s : w->streams)
      if (s) cudaStreamDestroy(s);
    for (cudaEvent_t e : w->events) cudaEventDestroy(e);
    for (cudaEvent_t e : w->tev) cudaEventDestroy(e);
    delete w;
  }
  t->workers.clear();
}

static WorkerState* worker_for_node(northup_tree_s* t, int node) {
  for (WorkerState* w : t->workers)
    if (w->node == node) return w;
  return nullptr;
}

// Make sure the HBM node's arena holds `bytes` (cudaMalloc on first use,
// grown when a larger plan arrives; counted in the node's `used`).
static int ensure_arena(northup_tree_s* t, int node, uint64_t bytes) {
  Node& n = t->nodes[node];
  if (bytes == 0 || n.arena_bytes >= bytes) return 0;
  if (n.arena && !n.arena_owned)
    return fail(NU_ENOMEM, "caller arena of node %d has %llu B, plan needs %llu B", node,
                (unsigned long long)n.arena_bytes, (unsigned long long)bytes);
  const uint64_t other = n.used - (n.arena_owned ? n.arena_bytes : 0);
  if (n.capacity && other + bytes > n.capacity)
    return fail(NU_ENOMEM, "node %d: plan needs %llu B, capacity %llu B (%llu in use)", node,
                (unsigned long long)bytes, (unsigned long long)n.capacity,
                (unsigned long long)other);
  cudaSetDevice(n.phys);
  if (n.arena) {
    cudaFree(n.arena);
    n.used -= n.arena_bytes;
    n.arena = nullptr;
    n.arena_bytes = 0;
  }
  cudaError_t e = cudaMalloc(&n.arena, bytes);
  if (e != cudaSuccess) {
    n.arena = nullptr;
    return fail(NU_ENOMEM, "cudaMalloc(%llu) for node %d arena: %s", (unsigned long long)bytes, node,
                cudaGetErrorString(e));
  }
  n.arena_bytes = bytes;
  n.arena_owned = true;
  n.used += bytes;
  return 0;
}

struct RunCtx {
  northup_tree_s* t;
  const Plan* plan;
  std::vector<char*> base;             // per plan buffer
  const std::vector<char>* needs_event;
  const northup_gemm_opts* o;
  bool timing;
};

static int run_worker(RunCtx& c, int wi, double* busy) {
  const Plan& P = *c.plan;
  WorkerState* w = worker_for_node(c.t, P.worker_node[wi]);
  if (!w) return fail(NU_ESTATE, "no worker state for node %d", P.worker_node[wi]);
  cudaError_t e = cudaSetDevice(w->device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
  const size_t nops = P.ops.size();
  while (w->events.size() < nops) {
    cudaEvent_t ev;
    e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_fail(e, "cudaEventCreate");
    w->events.push_back(ev);
  }
  if (c.timing) {
    while (w->tev.size() < 2 * nops) {
      cudaEvent_t ev;
      e = cudaEventCreate(&ev);
      if (e != cudaSuccess) return cuda_fail(e, "cudaEventCreate");
      w->tev.push_back(ev);
    }
  }
  for (size_t i = 0; i < nops; ++i) {
    const northup_op& op = P.ops[i];
    if (op.worker != wi) continue;
    cudaStream_t s = w->streams[op.stream];
    for (int d = 0; d < op.ndeps; ++d) {
      e = cudaStreamWaitEvent(s, w->events[op.deps[d]], 0);
      if (e != cudaSuccess) return cuda_fail(e, "cudaStreamWaitEvent");
    }
    if (c.timing) cudaEventRecord(w->tev[2 * i], s);
    if (op.op == NU_OP_COPY) {
      const char* src = c.base[op.src_buf] + op.src_off * 4;
      char* dst = c.base[op.dst_buf] + op.dst_off * 4;
      if (op.src_ld == op.cols && op.dst_ld == op.cols)
        e = cudaMemcpyAsync(dst, src, static_cast<size_t>(op.rows * op.cols) * 4, cudaMemcpyDefault, s);
      else
        e = cudaMemcpy2DAsync(dst, op.dst_ld * 4, src, op.src_ld * 4, op.cols * 4, op.rows,
                              cudaMemcpyDefault, s);
      if (e != cudaSuccess) return cuda_fail(e, "copy");
    } else if (op.op == NU_OP_LEAF) {
      const float* a = reinterpret_cast<const float*>(c.base[op.a_buf] + op.a_off * 4);
      const float* b = reinterpret_cast<const float*>(c.base[op.b_buf] + op.b_off * 4);
      float* cc = reinterpret_cast<float*>(c.base[op.c_buf] + op.c_off * 4);
      int rc = leaf_gemm_launch(a, op.lda, b, op.ldb, cc, op.ldc, op.m, op.n, op.k, op.accumulate,
                                P.kc, P.npass, s);
      if (rc) return rc;
    } else if (op.op == NU_OP_ZERO) {
      char* cc = c.base[op.c_buf] + op.c_off * 4;
      e = cudaMemset2DAsync(cc, op.ldc * 4, 0, op.n * 4, op.m, s);
      if (e != cudaSuccess) return cuda_fail(e, "memset");
    }
    if (c.timing) cudaEventRecord(w->tev[2 * i + 1], s);
    if ((*c.needs_event)[i]) {
      e = cudaEventRecord(w->events[i], s);
      if (e != cudaSuccess) return cuda_fail(e, "cudaEventRecord");
    }
  }
  for (cudaStream_t s : w->streams) {
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "stream synchronize");
  }
  if (c.timing) {
    for (size_t i = 0; i < nops; ++i) {
      const northup_op& op = P.ops[i];
      if (op.worker != wi) continue;
      float ms = 0.f;
      if (cudaEventElapsedTime(&ms, w->tev[2 * i], w->tev[2 * i + 1]) == cudaSuccess)
        busy[op.stream] += ms;
    }
  }
  return 0;
}

int execute_plan(northup_tree_s* t, const Plan& P, void* a, void* b, void* c,
                 const northup_gemm_opts* o, northup_stats* st) {
  RunCtx ctx;
  ctx.t = t;
  ctx.plan = &P;
  ctx.o = o;
  ctx.timing = o && o->collect_timing;
  ctx.base.resize(P.bufs.size(), nullptr);
  for (size_t i = 0; i < P.bufs.size(); ++i) {
    const PlanBuf& pb = P.bufs[i];
    switch (pb.kind) {
      case B_USER_A: ctx.base[i] = static_cast<char*>(a); break;
      case B_USER_B: ctx.base[i] = static_cast<char*>(b); break;
      case B_USER_C: ctx.base[i] = static_cast<char*>(c); break;
      default: {
        int rc = ensure_arena(t, pb.node, pb.bytes);
        if (rc) return rc;
        ctx.base[i] = static_cast<char*>(t->nodes[pb.node].arena);
      }
    }
  }
  // Only record an event where some later op on another stream waits for it.
  std::vector<char> needs(P.ops.size(), 0);
  for (const northup_op& op : P.ops)
    for (int d = 0; d < op.ndeps; ++d) needs[op.deps[d]] = 1;
  ctx.needs_event = &needs;

  const int W = P.num_workers;
  std::vector<int> rcs(W, 0);
  std::vector<std::vector<double>> busy(W, std::vector<double>(S_NUM, 0.0));
  std::string first_err;
  if (W == 1) {
    rcs[0] = run_worker(ctx, 0, busy[0].data());
    if (rcs[0]) first_err = northup_last_error();
  } else {
    std::vector<std::thread> th;
    std::vector<std::string> errs(W);
    for (int wi = 0; wi < W; ++wi)
      th.emplace_back([&, wi] {
        rcs[wi] = run_worker(ctx, wi, busy[wi].data());
        if (rcs[wi]) errs[wi] = northup_last_error();
      });
    for (auto& x : th) x.join();
    for (int wi = 0; wi < W; ++wi)
      if (rcs[wi] && first_err.empty()) first_err = errs[wi];
  }
  for (int wi = 0; wi < W; ++wi) {
    if (rcs[wi]) return fail(rcs[wi], "worker %d: %s", wi, first_err.c_str());
    if (st) {
      st->t_h2d_ms += busy[wi][S_H2D];
      st->t_compute_ms += busy[wi][S_COMP];
      st->t_d2h_ms += busy[wi][S_D2H] + busy[wi][S_D2D];
    }
  }
  return 0;
}

}  // namespace nu
