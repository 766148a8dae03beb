// Executor: runs a plan on the GPUs of the tree.
//
// One host worker thread per HBM sibling (branch parallelism, Fig. 2).
// Each worker owns CUDA streams for the edges of its subtree: H2D copies
// (data_down), the leaf kernel (compute_task), D2H copies (data_up) and D2D
// layout copies.  Ops are issued in plan order; each dependency on an op of
// another stream becomes a cudaStreamWaitEvent, so transfers of later
// chunks overlap the computation of earlier ones ("overlapping computation
// and communications (i.e. OpenCL/CUDA streams) at the leaf node").
//
// A FILE root adds a host I/O thread (file <-> DRAM staging, Listing 4):
//   CUDA op waiting for an I/O op  -> the worker thread blocks before issuing it
//   I/O op waiting for a CUDA op   -> the I/O thread waits until the op has been
//                                     issued, then cudaEventSynchronize.
// All dependencies point backwards in plan order, which every thread follows,
// so the waits cannot deadlock.
#include <ctype.h>
#include <errno.h>
#include <pthread.h>
#include <sched.h>
#include <stdio.h>
#include <fcntl.h>
#include <string.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <memory>
#include <mutex>
#include <thread>

#include <dlfcn.h>
#include <cstdio>

#include <deque>
#include <map>

#include "northup_internal.h"
#include "plan_builder.h"

struct WorkerState {
  int node = -1;
  int device = -1;
  cudaStream_t streams[nu::S_NUM] = {};
  std::vector<cudaEvent_t> events;       // one per op (reused across calls)
  std::vector<cudaEvent_t> tev;          // timing events (2 per op, timing mode)
};

namespace nu {

// CPUs of the NUMA node the GPU's PCIe device sits on (empty when the host
// does not say: one node, or numa_node = -1).
static std::vector<int> gpu_numa_cpus(int device) {
  std::vector<int> cpus;
  char bus[32] = {};
  if (cudaDeviceGetPCIBusId(bus, sizeof bus, device) != cudaSuccess) {
    cudaGetLastError();
    return cpus;
  }
  for (char* p = bus; *p; ++p) *p = static_cast<char>(tolower(*p));
  char path[128];
  snprintf(path, sizeof path, "/sys/bus/pci/devices/%s/numa_node", bus);
  FILE* f = fopen(path, "r");
  int node = -1;
  if (f) {
    if (fscanf(f, "%d", &node) != 1) node = -1;
    fclose(f);
  }
  if (node < 0) return cpus;
  snprintf(path, sizeof path, "/sys/devices/system/node/node%d/cpulist", node);
  f = fopen(path, "r");
  if (!f) return cpus;
  char list[4096] = {};
  if (fgets(list, sizeof list, f)) {
    for (char* tok = strtok(list, ",\n"); tok; tok = strtok(nullptr, ",\n")) {
      int lo = 0, hi = 0;
      if (sscanf(tok, "%d-%d", &lo, &hi) == 2)
        for (int c = lo; c <= hi; ++c) cpus.push_back(c);
      else if (sscanf(tok, "%d", &lo) == 1)
        cpus.push_back(lo);
    }
  }
  fclose(f);
  return cpus;
}

// each worker thread issues its GPU's copies from the CPUs of
// that GPU's NUMA node (bound at the start of every call).
void numa_bind_plan(northup_tree_s* t) {
  t->worker_cpus.assign(t->nodes.size(), {});
  if (getenv("NORTHUP_NO_NUMA_BIND")) return;
  for (WorkerState* w : t->workers) t->worker_cpus[w->node] = gpu_numa_cpus(w->device);
}

void bind_worker_thread(const northup_tree_s* t, int node) {
  if (node < 0 || node >= static_cast<int>(t->worker_cpus.size()) || t->worker_cpus[node].empty()) return;
  cpu_set_t set;
  CPU_ZERO(&set);
  for (int c : t->worker_cpus[node])
    if (c >= 0 && c < CPU_SETSIZE) CPU_SET(c, &set);
  pthread_setaffinity_np(pthread_self(), sizeof set, &set);
}

// The planner's PCIe term (S§8(d) "BW_e = the concurrently measured per-GPU
// bandwidth with all links active"): every local GPU copies 128 MiB H2D and
// 128 MiB D2H at once, one warm-up round and four timed ones; each GPU's best
// H2D rate (a single short round once read 27 instead of ~50 GB/s on a box,
// and the planner then chose a much worse S2B split), the slowest GPU's.
// Skipped for HBM roots (no host edge) and with NORTHUP_CALIBRATE=0.
int calibrate_pcie(northup_tree_s* t) {
  t->pcie_gbs = 0.0;
  const char* env = getenv("NORTHUP_CALIBRATE");
  if ((env && env[0] == '0') || t->workers.empty() || t->nodes[0].storage == NU_HBM) return 0;
  const size_t bytes = 128ull << 20;
  const size_t W = t->workers.size();
  std::vector<void*> hin(W, nullptr), hout(W, nullptr), din(W, nullptr), dout(W, nullptr);
  std::vector<cudaEvent_t> ev(4 * W, nullptr);
  int rc = 0;
  for (size_t i = 0; i < W && !rc; ++i) {
    cudaSetDevice(t->workers[i]->device);
    if (cudaHostAlloc(&hin[i], bytes, cudaHostAllocPortable) != cudaSuccess ||
        cudaHostAlloc(&hout[i], bytes, cudaHostAllocPortable) != cudaSuccess ||
        cudaMalloc(&din[i], bytes) != cudaSuccess || cudaMalloc(&dout[i], bytes) != cudaSuccess)
      rc = 1;
    for (int k = 0; k < 4 && !rc; ++k)
      if (cudaEventCreate(&ev[4 * i + k]) != cudaSuccess) rc = 1;
  }
  std::vector<double> best(W, 0.0);
  for (int round = 0; round < 5 && !rc; ++round) {
    for (size_t i = 0; i < W; ++i) {
      WorkerState* w = t->workers[i];
      cudaSetDevice(w->device);
      cudaEventRecord(ev[4 * i + 0], w->streams[S_H2D]);
      cudaMemcpyAsync(din[i], hin[i], bytes, cudaMemcpyHostToDevice, w->streams[S_H2D]);
      cudaEventRecord(ev[4 * i + 1], w->streams[S_H2D]);
      cudaEventRecord(ev[4 * i + 2], w->streams[S_D2H]);
      cudaMemcpyAsync(hout[i], dout[i], bytes, cudaMemcpyDeviceToHost, w->streams[S_D2H]);
      cudaEventRecord(ev[4 * i + 3], w->streams[S_D2H]);
    }
    for (size_t i = 0; i < W; ++i) {
      cudaSetDevice(t->workers[i]->device);
      float ms = 0.f;
      if (cudaEventSynchronize(ev[4 * i + 1]) != cudaSuccess ||
          cudaEventElapsedTime(&ms, ev[4 * i + 0], ev[4 * i + 1]) != cudaSuccess || ms <= 0.f) {
        rc = 1;
        break;
      }
      if (round > 0) best[i] = std::max(best[i], bytes / (ms * 1e-3) / 1e9);   // round 0: warm-up
      cudaEventSynchronize(ev[4 * i + 3]);
    }
  }
  double worst = rc || W == 0 ? 0.0 : *std::min_element(best.begin(), best.end());
  for (size_t i = 0; i < W; ++i) {
    cudaSetDevice(t->workers[i]->device);
    if (hin[i]) cudaFreeHost(hin[i]);
    if (hout[i]) cudaFreeHost(hout[i]);
    if (din[i]) cudaFree(din[i]);
    if (dout[i]) cudaFree(dout[i]);
    for (int k = 0; k < 4; ++k)
      if (ev[4 * i + k]) cudaEventDestroy(ev[4 * i + k]);
  }
  cudaGetLastError();
  if (!rc && worst > 1.0 && worst < 1e6) t->pcie_gbs = worst;
  return 0;   // calibration is best effort: the planner falls back to its constant
}

int finalize_workers(northup_tree_s* t) {
  int ndev = northup_device_count();
  for (const Node& n : t->nodes) {
    if (n.storage != NU_HBM) continue;
    if (t->local_node >= 0 && n.id != t->local_node) continue;   // run by a peer process
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
    // load every kernel now: with lazy module loading a kernel's first launch can
    // block the issuing thread behind a stream that waits on another worker's or
    // process's progress (cross-sibling waits), which can close a cycle
    preload_kernels();
  }
  // Shared staging pulls panels from sibling HBM: it is planned only when
  // every pair of distinct HBM devices (local or in peer processes) has P2P
  // access; enable it between the local ones.
  t->p2p_ok = true;
  for (const Node& a : t->nodes)
    for (const Node& b : t->nodes) {
      if (a.storage != NU_HBM || b.storage != NU_HBM || a.phys == b.phys) continue;
      int can = 0;
      if (cudaDeviceCanAccessPeer(&can, a.phys, b.phys) != cudaSuccess || !can) t->p2p_ok = false;
    }
  cudaGetLastError();
  for (WorkerState* a : t->workers)
    for (WorkerState* b : t->workers) {
      if (a->device == b->device) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, a->device, b->device);
      if (!can) continue;
      cudaSetDevice(a->device);
      cudaError_t e = cudaDeviceEnablePeerAccess(b->device, 0);
      if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
      else if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceEnablePeerAccess");
    }
  numa_bind_plan(t);
  return calibrate_pcie(t);
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
int ensure_arena(northup_tree_s* t, int node, uint64_t bytes) {
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
  if (n.storage == NU_HOST) {
    if (n.arena) {
      cudaFreeHost(n.arena);
      n.used -= n.arena_bytes;
      n.arena = nullptr;
      n.arena_bytes = 0;
    }
    cudaError_t e = cudaHostAlloc(&n.arena, bytes, cudaHostAllocPortable);
    if (e != cudaSuccess) {
      n.arena = nullptr;
      return fail(NU_ENOMEM, "cudaHostAlloc(%llu) for staging node %d: %s", (unsigned long long)bytes,
                  node, cudaGetErrorString(e));
    }
  } else {
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
      return fail(NU_ENOMEM, "cudaMalloc(%llu) for node %d arena: %s", (unsigned long long)bytes,
                  node, cudaGetErrorString(e));
    }
  }
  n.arena_bytes = bytes;
  n.arena_owned = true;
  n.used += bytes;
  return 0;
}

struct RunCtx {
  northup_tree_s* t;
  const Plan* plan;
  std::vector<char*> base;             // per plan buffer (host/device pointers)
  std::vector<const northup_buf_s*> file;   // per plan buffer: file handle or NULL
  const std::vector<char>* needs_event;
  const std::vector<uint64_t>* needs_remote;   // per local op: mask of sibling processes waiting
  const northup_gemm_opts* o;
  bool timing;
  int local = -1;                          // multi-process siblings: the local worker
  bool cross = false;                      // the plan has cross-sibling dependencies
  uint32_t gen = 0;
  // cross-thread progress (FILE roots)
  std::mutex m;
  std::condition_variable cv;
  std::vector<char> issued;            // CUDA op: event recorded
  std::vector<char> io_done;           // I/O op: finished
  std::atomic<bool> abort{false};
  double io_ms = 0;
  int io_mode = 0;                     // file <-> HBM: 1 = cuFile, 2 = pinned bounce
};

static void mark(RunCtx& c, std::vector<char>& v, size_t i) {
  {
    std::lock_guard<std::mutex> g(c.m);
    v[i] = 1;
  }
  c.cv.notify_all();
}

// Wait until flag i is set (or the run aborted).  Returns false on abort.
static bool wait_flag(RunCtx& c, std::vector<char>& v, size_t i) {
  std::unique_lock<std::mutex> g(c.m);
  c.cv.wait(g, [&] { return v[i] || c.abort.load(); });
  return v[i] != 0;
}

static int run_worker(RunCtx& c, int wi, double* busy, cudaGraphExec_t* capture_out = nullptr) {
  const Plan& P = *c.plan;
  WorkerState* w = worker_for_node(c.t, P.worker_node[wi]);
  if (!w) return fail(NU_ESTATE, "no worker state for node %d", P.worker_node[wi]);
  cudaError_t e = cudaSetDevice(w->device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
  cudaEvent_t fork = nullptr;
  if (capture_out) {
    // Stream capture: stream 0 starts the capture, the other streams join it
    // through a fork event and are joined back at the end, so the graph holds
    // every op with its cross-stream dependencies.
    e = cudaStreamBeginCapture(w->streams[0], cudaStreamCaptureModeThreadLocal);
    if (e != cudaSuccess) return cuda_fail(e, "cudaStreamBeginCapture");
    cudaEventCreateWithFlags(&fork, cudaEventDisableTiming);
    cudaEventRecord(fork, w->streams[0]);
    for (int s = 1; s < S_NUM; ++s) cudaStreamWaitEvent(w->streams[s], fork, 0);
  }
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
  const bool dbg = getenv("NORTHUP_DEBUG_EXEC") != nullptr;
  for (size_t i = 0; i < nops; ++i) {
    const northup_op& op = P.ops[i];
    if (op.worker != wi) continue;
    cudaStream_t s = w->streams[op.stream];
    if (dbg) fprintf(stderr, "[northup] worker %d issues op %zu (kind %d, stream %d, %d deps)\n", wi, i, op.op,
                     op.stream, op.ndeps);
    for (int d = 0; d < op.ndeps; ++d) {
      const northup_op& q = P.ops[op.deps[d]];
      if (is_io_stream(q.stream)) {
        if (!wait_flag(c, c.io_done, op.deps[d])) return fail(NU_EIO, "aborted: file I/O failed");
        continue;
      }
      cudaEvent_t ev = w->events[op.deps[d]];
      if (q.worker != wi && c.local >= 0) {
        // a sibling in another process: device-side wait on its flag word
        // a sibling in another process: device-side wait on OUR flag word for
        // that op, which the producer writes remotely after the op
        int rc = stream_wait_flag(s, c.t->flags + P.num_workers + op.deps[d], c.gen);
        if (rc) return rc;
        continue;
      }
      if (q.worker != wi) {
        // another sibling's op (shared-staging pull, NEXT-1): wait until that
        // worker has recorded its event in this call, then wait on it on the
        // device (cross-device event waits are legal).  Dependencies point
        // backwards in plan order, so this cannot deadlock.
        if (!wait_flag(c, c.issued, op.deps[d])) return fail(NU_ECUDA, "aborted: a sibling worker failed");
        ev = worker_for_node(c.t, P.worker_node[q.worker])->events[op.deps[d]];
      }
      e = cudaStreamWaitEvent(s, ev, 0);
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
      int slow_pct = 0;
      if (debug_slow_sibling(&slow_pct) == wi && slow_pct > 0) debug_spin(debug_slow_ns(slow_pct, op.m, op.n, op.k), s);
      const float* a = reinterpret_cast<const float*>(c.base[op.a_buf] + op.a_off * 4);
      const float* b = reinterpret_cast<const float*>(c.base[op.b_buf] + op.b_off * 4);
      float* cc = reinterpret_cast<float*>(c.base[op.c_buf] + op.c_off * 4);
      LeafCall lc{};
      lc.A = a, lc.lda = op.lda, lc.B = b, lc.ldb = op.ldb, lc.C = cc, lc.ldc = op.ldc;
      lc.M = op.m, lc.N = op.n, lc.K = op.k, lc.accumulate = op.accumulate, lc.panel = P.kc, lc.npass = P.npass;
      if (op.src_buf >= 0) {   // B split in place by earlier NU_OP_SPLIT_B ops
        lc.eb_presplit = reinterpret_cast<const int*>(c.base[op.src_buf] + op.src_off * 4);
        lc.eb_stride = op.rows;
      }
      if (wi < static_cast<int>(P.scr_buf.size()) && P.scr_buf[wi] >= 0) {
        lc.scratch = c.base[P.scr_buf[wi]] + P.scr_off[wi];
        lc.scratch_bytes = P.scr_bytes[wi];
      }
      lc.stream = s;
      int rc = leaf_run(lc);
      if (rc) return rc;
    } else if (op.op == NU_OP_SPLIT_B) {
      if (wi >= static_cast<int>(P.scr_buf.size()) || P.scr_buf[wi] < 0)
        return fail(NU_ESTATE, "split op without a leaf scratch");
      float* bp = reinterpret_cast<float*>(c.base[op.dst_buf] + op.dst_off * 4);
      int* eb = reinterpret_cast<int*>(c.base[op.c_buf] + op.c_off * 4);
      unsigned* bmax = reinterpret_cast<unsigned*>(c.base[P.scr_buf[wi]] + P.scr_off[wi]);
      int rc = leaf::split_b_launch(bp, op.dst_ld, static_cast<int>(op.rows), static_cast<int>(op.cols), bp,
                                    op.dst_ld, eb, bmax, s);
      if (rc) return rc;
    } else if (op.op == NU_OP_STENCIL) {
      const float* tin = reinterpret_cast<const float*>(c.base[op.a_buf] + op.a_off * 4);
      const float* pw = reinterpret_cast<const float*>(c.base[op.b_buf] + op.b_off * 4);
      float* tout = reinterpret_cast<float*>(c.base[op.c_buf] + op.c_off * 4);
      int rc = hotspot_launch(tin, op.lda, pw, op.ldb, tout, op.ldc, op.m, op.n, op.src_off, op.dst_off,
                              op.rows, op.cols, static_cast<int>(op.k), P.hs_coef, s);
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
      mark(c, c.issued, i);
    }
    if (c.local >= 0 && (*c.needs_remote)[i]) {
      // publish op i to every sibling process that waits for it: a fenced
      // remote store into its flag words (consumers only ever poll local memory)
      const uint64_t mask = (*c.needs_remote)[i];
      for (int q = 0; q < P.num_workers; ++q)
        if (mask >> q & 1) {
          int rc = stream_write_flag(s, c.t->peers[q].flags + P.num_workers + i, c.gen);
          if (rc) return rc;
        }
    }
  }
  if (c.local >= 0 && c.cross) {
    // device-side join: done word after all local streams, then wait for every
    // sibling's done word, so no peer still reads this arena when we return
    for (int k = 1; k < S_NUM; ++k) {
      cudaEvent_t j = nullptr;
      e = cudaEventCreateWithFlags(&j, cudaEventDisableTiming);
      if (e != cudaSuccess) return cuda_fail(e, "cudaEventCreate");
      cudaEventRecord(j, w->streams[k]);
      cudaStreamWaitEvent(w->streams[0], j, 0);
      cudaEventDestroy(j);
    }
    int rc = 0;
    for (int q = 0; q < P.num_workers && !rc; ++q)
      if (q != wi) rc = stream_write_flag(w->streams[0], c.t->peers[q].flags + wi, c.gen);
    for (int q = 0; q < P.num_workers && !rc; ++q)
      if (q != wi) rc = stream_wait_flag(w->streams[0], c.t->flags + q, c.gen);
    if (rc) return rc;
  }
  if (capture_out) {
    std::vector<cudaEvent_t> joins;
    for (int s = 1; s < S_NUM; ++s) {
      cudaEvent_t j;
      cudaEventCreateWithFlags(&j, cudaEventDisableTiming);
      cudaEventRecord(j, w->streams[s]);
      cudaStreamWaitEvent(w->streams[0], j, 0);
      joins.push_back(j);
    }
    cudaGraph_t g = nullptr;
    e = cudaStreamEndCapture(w->streams[0], &g);
    for (cudaEvent_t j : joins) cudaEventDestroy(j);
    cudaEventDestroy(fork);
    if (e != cudaSuccess) return cuda_fail(e, "cudaStreamEndCapture");
    e = cudaGraphInstantiate(capture_out, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGraphInstantiate");
    e = cudaGraphLaunch(*capture_out, w->streams[0]);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGraphLaunch");
  }
  if (c.local >= 0 && c.cross) {
    // multi-process siblings: the streams wait on flags other processes write, so a
    // peer that died would block them forever; poll with a deadline instead
    // (NORTHUP_PEER_TIMEOUT_S, default 600 s) and fail loudly
    const char* to = getenv("NORTHUP_PEER_TIMEOUT_S");
    const double limit = to ? atof(to) : 600.0;
    const auto t0 = std::chrono::steady_clock::now();
    if (dbg) fprintf(stderr, "[northup] worker %d: all ops issued, polling (limit %.0f s)\n", wi, limit);
    for (cudaStream_t s : w->streams) {
      while ((e = cudaStreamQuery(s)) == cudaErrorNotReady) {
        if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > limit)
          return fail(NU_ECUDA, "multi-process siblings: no progress from the peer processes for %.0f s "
                                "(did a sibling fail?)", limit);
        std::this_thread::sleep_for(std::chrono::microseconds(20));
      }
      if (e != cudaSuccess) return cuda_fail(e, "stream synchronize");
    }
  }
  for (cudaStream_t s : w->streams) {
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "stream synchronize");
  }
  if (c.timing) {
    // per-op (start, end) relative to this worker's first op, for the timeline
    int first = -1;
    for (size_t i = 0; i < nops; ++i)
      if (P.ops[i].worker == wi) {
        first = static_cast<int>(i);
        break;
      }
    for (size_t i = 0; i < nops; ++i) {
      const northup_op& op = P.ops[i];
      if (op.worker != wi) continue;
      float ms = 0.f, t0 = 0.f, t1 = 0.f;
      if (cudaEventElapsedTime(&ms, w->tev[2 * i], w->tev[2 * i + 1]) == cudaSuccess)
        busy[op.stream] += ms;
      cudaEventElapsedTime(&t0, w->tev[2 * first], w->tev[2 * i]);
      cudaEventElapsedTime(&t1, w->tev[2 * first], w->tev[2 * i + 1]);
      std::lock_guard<std::mutex> g(c.m);
      c.t->timeline.push_back({static_cast<float>(i), static_cast<float>(wi),
                               static_cast<float>(op.stream), t0, t1});
    }
  }
  return 0;
}

// Positional file I/O of a rows x cols fp32 block (element offsets / leading
// dimensions); O_DIRECT when the file has a direct descriptor and
// buffer, offset and length are 4 KiB aligned, else buffered I/O.
static int file_block(const northup_buf_s* f, bool write, char* mem, int64_t mem_ld,
                      int64_t file_off, int64_t file_ld, int64_t rows, int64_t cols) {
  auto io = [&](char* p, uint64_t bytes, uint64_t off) -> int {
    int fd = f->fd;
    if (f->direct_fd >= 0 && reinterpret_cast<uintptr_t>(p) % 4096 == 0 && bytes % 4096 == 0 &&
        off % 4096 == 0)
      fd = f->direct_fd;
    while (bytes) {
      ssize_t r = pio(fd, p, bytes, off, write);
      if (r < 0) {
        if (errno == EINTR) continue;
        const int err = errno;
        note_io_errno(err);
        return fail(NU_EIO, "%s(%s): %s", write ? "pwrite" : "pread", f->path.c_str(), strerror(err));
      }
      if (r == 0) {
        note_io_errno(0);
        return fail(NU_EIO, "%s(%s): short transfer", write ? "pwrite" : "pread", f->path.c_str());
      }
      p += r;
      bytes -= static_cast<uint64_t>(r);
      off += static_cast<uint64_t>(r);
    }
    return 0;
  };
  if (mem_ld == cols && file_ld == cols)
    return io(mem, static_cast<uint64_t>(rows * cols) * 4, static_cast<uint64_t>(file_off) * 4);
  for (int64_t r = 0; r < rows; ++r) {
    int rc = io(mem + r * mem_ld * 4, static_cast<uint64_t>(cols) * 4,
                static_cast<uint64_t>(file_off + r * file_ld) * 4);
    if (rc) return rc;
  }
  return 0;
}

// ---- FILE <-> HBM directly (the GDS edge, NEXT-4) -------------------------
// cuFile (GPUDirect Storage) is loaded with dlopen so the library does not
// depend on it.  Where the file system has no GDS support cuFile runs in its
// compat mode (/etc/cufile.json allow_compat_mode); if the driver cannot be
// opened at all, transfers bounce through a pinned host buffer.
namespace {
struct CuFileApi {
  bool tried = false, ok = false, timed_out = false;
  struct Err {
    int err;
    int cu_err;
  };
  Err (*driver_open)() = nullptr;
  Err (*handle_register)(void**, void*) = nullptr;
  void (*handle_deregister)(void*) = nullptr;
  ssize_t (*read)(void*, void*, size_t, off_t, off_t) = nullptr;
  ssize_t (*write)(void*, const void*, size_t, off_t, off_t) = nullptr;
};
CuFileApi g_cufile;
std::mutex g_cufile_m;

CuFileApi& cufile() {
  std::lock_guard<std::mutex> g(g_cufile_m);
  if (g_cufile.tried) return g_cufile;
  g_cufile.tried = true;
  // opt-in: cuFile's compat mode hung on this pool's boxes (virtio disk, no
  // nvidia-fs), so the pinned bounce is the default and NORTHUP_CUFILE=1 asks
  // for GPUDirect Storage
  const char* want = getenv("NORTHUP_CUFILE");
  if (!want || want[0] != '1') return g_cufile;
  const bool dbg = getenv("NORTHUP_CUFILE_DEBUG") != nullptr;
  void* h = dlopen("libcufile.so.0", RTLD_NOW | RTLD_LOCAL);
  if (!h) h = dlopen("libcufile.so", RTLD_NOW | RTLD_LOCAL);
  if (!h) return g_cufile;
  g_cufile.driver_open = reinterpret_cast<CuFileApi::Err (*)()>(dlsym(h, "cuFileDriverOpen"));
  g_cufile.handle_register = reinterpret_cast<CuFileApi::Err (*)(void**, void*)>(dlsym(h, "cuFileHandleRegister"));
  g_cufile.handle_deregister = reinterpret_cast<void (*)(void*)>(dlsym(h, "cuFileHandleDeregister"));
  g_cufile.read = reinterpret_cast<ssize_t (*)(void*, void*, size_t, off_t, off_t)>(dlsym(h, "cuFileRead"));
  g_cufile.write = reinterpret_cast<ssize_t (*)(void*, const void*, size_t, off_t, off_t)>(dlsym(h, "cuFileWrite"));
  if (!g_cufile.driver_open || !g_cufile.handle_register || !g_cufile.read || !g_cufile.write) return g_cufile;
  if (dbg) fprintf(stderr, "[northup] cuFileDriverOpen ...\n");
  // Watchdog: cuFileDriverOpen has hung on boxes without nvidia-fs; run it on a
  // detached thread and give up after NORTHUP_CUFILE_TIMEOUT_S (default 20 s),
  // falling back to the pinned bounce instead of blocking the caller forever.
  struct OpenState {
    std::mutex m;
    std::condition_variable cv;
    bool done = false, ok = false;
  };
  auto st = std::make_shared<OpenState>();
  auto open_fn = g_cufile.driver_open;
  std::thread([st, open_fn] {
    const bool ok = open_fn().err == 0;
    std::lock_guard<std::mutex> g(st->m);
    st->done = true;
    st->ok = ok;
    st->cv.notify_all();
  }).detach();
  const char* to = getenv("NORTHUP_CUFILE_TIMEOUT_S");
  const double secs = (to && atof(to) > 0) ? atof(to) : 20.0;
  {
    std::unique_lock<std::mutex> lk(st->m);
    st->cv.wait_for(lk, std::chrono::duration<double>(secs), [&] { return st->done; });
    g_cufile.ok = st->done && st->ok;
    g_cufile.timed_out = !st->done;
  }
  if (dbg)
    fprintf(stderr, "[northup] cuFileDriverOpen -> %s\n",
            g_cufile.ok ? "ok" : (g_cufile.timed_out ? "timed out (pinned bounce)" : "failed"));
  return g_cufile;
}

// CUfileDescr_t as in cufile.h: type, union {int fd; void* handle;}, fs_ops.
struct CuFileDescr {
  int type;
  union {
    int fd;
    void* handle;
  } h;
  const void* fs_ops;
};
}  // namespace

struct DevIO {
  std::map<const northup_buf_s*, void*> handles;   // cuFile handle per file
  char* bounce = nullptr;                          // pinned fallback buffer: two halves
  size_t bounce_bytes = 0;
  int mode = 0;                                    // 1 = cuFile, 2 = bounce
  struct Dev {
    cudaStream_t s = nullptr;
    cudaEvent_t ev[2] = {nullptr, nullptr};
  };
  std::map<int, Dev> dev;                          // copy stream + per-half events per device
  ~DevIO() {
    for (auto& kv : handles)
      if (kv.second && g_cufile.handle_deregister) g_cufile.handle_deregister(kv.second);
    for (auto& kv : dev) {
      cudaSetDevice(kv.first);
      if (kv.second.s) cudaStreamSynchronize(kv.second.s), cudaStreamDestroy(kv.second.s);
      for (cudaEvent_t e : kv.second.ev)
        if (e) cudaEventDestroy(e);
    }
    if (bounce) cudaFreeHost(bounce);
  }
};

// The pinned-bounce transfer of a rows x cols block between a file and device
// memory, pipelined over the two halves of the bounce buffer: while the DMA
// engine copies one group of rows (cudaMemcpy2DAsync on a private stream), the
// I/O thread reads (or writes) the next group from (to) the file.
static int bounce_block_dev(DevIO& io, const northup_buf_s* f, bool write, char* dmem, int64_t mem_ld,
                            int64_t file_off, int64_t file_ld, int64_t rows, int64_t cols) {
  io.mode = 2;
  if (!io.bounce) {
    io.bounce_bytes = 64ull << 20;
    cudaError_t e = cudaHostAlloc(reinterpret_cast<void**>(&io.bounce), io.bounce_bytes, cudaHostAllocPortable);
    if (e != cudaSuccess) return cuda_fail(e, "bounce buffer");
  }
  int d = 0;
  cudaGetDevice(&d);
  DevIO::Dev& D = io.dev[d];
  if (!D.s) {
    cudaError_t e = cudaStreamCreateWithFlags(&D.s, cudaStreamNonBlocking);
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) e = cudaEventCreateWithFlags(&D.ev[i], cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_fail(e, "bounce stream");
  }
  const uint64_t half = io.bounce_bytes / 2, row_bytes = static_cast<uint64_t>(cols) * 4;
  if (row_bytes > half) {   // one row larger than a half: split the columns
    for (int64_t c0 = 0; c0 < cols; c0 += static_cast<int64_t>(half / 4)) {
      const int64_t nc = std::min<int64_t>(static_cast<int64_t>(half / 4), cols - c0);
      int rc = bounce_block_dev(io, f, write, dmem + c0 * 4, mem_ld, file_off + c0, file_ld, rows, nc);
      if (rc) return rc;
    }
    return 0;
  }
  const int64_t per = static_cast<int64_t>(half / row_bytes);
  const int64_t ngroups = (rows + per - 1) / per;
  auto group = [&](int64_t g, int64_t* r0, int64_t* nr) {
    *r0 = g * per;
    *nr = std::min(per, rows - *r0);
  };
  cudaError_t e = cudaSuccess;
  if (!write) {
    for (int64_t g = 0; g < ngroups; ++g) {
      int64_t r0, nr;
      group(g, &r0, &nr);
      const int sl = static_cast<int>(g & 1);
      char* hb = io.bounce + sl * half;
      if ((e = cudaEventSynchronize(D.ev[sl])) != cudaSuccess) return cuda_fail(e, "bounce wait");
      int rc = file_block(f, false, hb, cols, file_off + r0 * file_ld, file_ld, nr, cols);
      if (rc) return rc;
      e = cudaMemcpy2DAsync(dmem + r0 * mem_ld * 4, static_cast<size_t>(mem_ld) * 4, hb, row_bytes, row_bytes,
                            static_cast<size_t>(nr), cudaMemcpyHostToDevice, D.s);
      if (e == cudaSuccess) e = cudaEventRecord(D.ev[sl], D.s);
      if (e != cudaSuccess) return cuda_fail(e, "bounce H2D");
    }
  } else {
    for (int64_t g = 0; g <= ngroups; ++g) {
      if (g < ngroups) {   // start the D2H of group g ...
        int64_t r0, nr;
        group(g, &r0, &nr);
        const int sl = static_cast<int>(g & 1);
        char* hb = io.bounce + sl * half;
        e = cudaMemcpy2DAsync(hb, row_bytes, dmem + r0 * mem_ld * 4, static_cast<size_t>(mem_ld) * 4, row_bytes,
                              static_cast<size_t>(nr), cudaMemcpyDeviceToHost, D.s);
        if (e == cudaSuccess) e = cudaEventRecord(D.ev[sl], D.s);
        if (e != cudaSuccess) return cuda_fail(e, "bounce D2H");
      }
      if (g > 0) {         // ... while group g - 1 goes to the file
        int64_t r0, nr;
        group(g - 1, &r0, &nr);
        const int sl = static_cast<int>((g - 1) & 1);
        if ((e = cudaEventSynchronize(D.ev[sl])) != cudaSuccess) return cuda_fail(e, "bounce wait");
        int rc = file_block(f, true, io.bounce + sl * half, cols, file_off + r0 * file_ld, file_ld, nr, cols);
        if (rc) return rc;
      }
    }
  }
  if ((e = cudaStreamSynchronize(D.s)) != cudaSuccess) return cuda_fail(e, "bounce sync");
  return 0;
}

// A rows x cols fp32 block between a file and DEVICE memory.
static int file_block_dev(DevIO& io, const northup_buf_s* f, bool write, char* dmem, int64_t mem_ld,
                          int64_t file_off, int64_t file_ld, int64_t rows, int64_t cols) {
  CuFileApi& api = cufile();
  void* fh = nullptr;
  if (api.ok) {
    auto it = io.handles.find(f);
    if (it == io.handles.end()) {
      CuFileDescr d{};
      d.type = 1;   // CU_FILE_HANDLE_TYPE_OPAQUE_FD
      d.h.fd = f->direct_fd >= 0 ? f->direct_fd : f->fd;
      void* h = nullptr;
      if (getenv("NORTHUP_CUFILE_DEBUG")) fprintf(stderr, "[northup] cuFileHandleRegister(fd %d) ...\n", d.h.fd);
      if (api.handle_register(&h, &d).err != 0) h = nullptr;
      if (getenv("NORTHUP_CUFILE_DEBUG")) fprintf(stderr, "[northup] cuFileHandleRegister -> %p\n", h);
      it = io.handles.emplace(f, h).first;
    }
    fh = it->second;
  }
  if (!fh) return bounce_block_dev(io, f, write, dmem, mem_ld, file_off, file_ld, rows, cols);
  auto xfer = [&](char* p, uint64_t bytes, uint64_t off) -> int {
    io.mode = 1;
    if (getenv("NORTHUP_CUFILE_DEBUG"))
      fprintf(stderr, "[northup] cuFile%s %llu B at %llu\n", write ? "Write" : "Read", (unsigned long long)bytes,
              (unsigned long long)off);
    while (bytes) {
      const ssize_t r = write ? api.write(fh, p, bytes, static_cast<off_t>(off), 0)
                              : api.read(fh, p, bytes, static_cast<off_t>(off), 0);
      if (r <= 0) return fail(NU_EIO, "cuFile%s(%s) returned %zd", write ? "Write" : "Read", f->path.c_str(), r);
      p += r;
      bytes -= static_cast<uint64_t>(r);
      off += static_cast<uint64_t>(r);
    }
    return 0;
  };
  if (mem_ld == cols && file_ld == cols)
    return xfer(dmem, static_cast<uint64_t>(rows * cols) * 4, static_cast<uint64_t>(file_off) * 4);
  for (int64_t r = 0; r < rows; ++r) {
    int rc = xfer(dmem + r * mem_ld * 4, static_cast<uint64_t>(cols) * 4,
                  static_cast<uint64_t>(file_off + r * file_ld) * 4);
    if (rc) return rc;
  }
  return 0;
}

// One I/O queue (`queue` = S_IO file reads or S_IOW file writes) on its own
// host thread, so a round's C write-back overlaps the next round's panel reads.
static int run_io(RunCtx& c, int queue) {
  const Plan& P = *c.plan;
  const auto t0 = std::chrono::steady_clock::now();
  DevIO dio;
  for (size_t i = 0; i < P.ops.size(); ++i) {
    const northup_op& op = P.ops[i];
    if (op.stream != queue) continue;
    for (int d = 0; d < op.ndeps; ++d) {
      const northup_op& q = P.ops[op.deps[d]];
      if (is_io_stream(q.stream)) {   // the other I/O queue (this one runs in order)
        if (q.stream != queue && !wait_flag(c, c.io_done, op.deps[d]))
          return fail(NU_EIO, "aborted: file I/O failed");
        continue;
      }
      if (!wait_flag(c, c.issued, op.deps[d])) return fail(NU_ECUDA, "aborted: a GPU worker failed");
      WorkerState* w = worker_for_node(c.t, P.worker_node[q.worker]);
      cudaSetDevice(w->device);
      cudaError_t e = cudaEventSynchronize(w->events[op.deps[d]]);
      if (e != cudaSuccess) return cuda_fail(e, "cudaEventSynchronize (I/O thread)");
    }
    int rc;
    // memory side in HBM (FILE -> HBM edge) or in host DRAM (staging)
    const int mb = op.op == NU_OP_IO_READ ? op.dst_buf : op.src_buf;
    const bool dev = P.bufs[mb].kind == B_ARENA && c.t->nodes[P.bufs[mb].node].storage == NU_HBM;
    if (dev) cudaSetDevice(c.t->nodes[P.bufs[mb].node].phys);
    if (op.op == NU_OP_IO_READ)
      rc = dev ? file_block_dev(dio, c.file[op.src_buf], false, c.base[op.dst_buf] + op.dst_off * 4, op.dst_ld,
                                op.src_off, op.src_ld, op.rows, op.cols)
               : file_block(c.file[op.src_buf], false, c.base[op.dst_buf] + op.dst_off * 4, op.dst_ld,
                            op.src_off, op.src_ld, op.rows, op.cols);
    else
      rc = dev ? file_block_dev(dio, c.file[op.dst_buf], true, c.base[op.src_buf] + op.src_off * 4, op.src_ld,
                                op.dst_off, op.dst_ld, op.rows, op.cols)
               : file_block(c.file[op.dst_buf], true, c.base[op.src_buf] + op.src_off * 4, op.src_ld,
                            op.dst_off, op.dst_ld, op.rows, op.cols);
    if (rc) return rc;
    mark(c, c.io_done, i);
  }
  // O_SYNC semantics of P:242: C is durable when northup_gemm returns.
  if (queue == S_IOW)
    for (size_t b = 0; b < c.file.size(); ++b)
      if (c.file[b] && P.bufs[b].kind == B_USER_C && fdatasync(c.file[b]->fd) != 0) {
        const int err = errno;
        note_io_errno(err);
        return fail(NU_EIO, "fdatasync(%s): %s", c.file[b]->path.c_str(), strerror(err));
      }
  const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  {
    std::lock_guard<std::mutex> g(c.m);
    c.io_ms = std::max(c.io_ms, ms);
    c.io_mode = std::max(c.io_mode, dio.mode);
  }
  return 0;
}

// Key of a captured GEMM: everything the op list and its pointers depend on.
static std::vector<int64_t> graph_key(const Plan& P, const std::vector<char*>& base,
                                      const northup_gemm_opts* o) {
  std::vector<int64_t> k = {P.M, P.N, P.K, P.kc, P.npass, o ? o->schedule : 0,
                            static_cast<int64_t>(P.ops.size())};
  for (char* b : base) k.push_back(reinterpret_cast<int64_t>(b));
  return k;
}

void destroy_graphs(northup_tree_s* t) {
  for (auto& g : t->graph_execs)
    if (g) cudaGraphExecDestroy(static_cast<cudaGraphExec_t>(g));
  t->graph_execs.clear();
  t->graph_key.clear();
}

int execute_plan(northup_tree_s* t, const Plan& P, northup_buf_s* a, northup_buf_s* b,
                 northup_buf_s* c, const northup_gemm_opts* o, northup_stats* st) {
  RunCtx ctx;
  ctx.t = t;
  ctx.plan = &P;
  ctx.o = o;
  ctx.timing = o && o->collect_timing;
  ctx.base.resize(P.bufs.size(), nullptr);
  ctx.file.resize(P.bufs.size(), nullptr);
  const int lw = local_worker(t, P);
  if (lw == -2) return fail(NU_ESTATE, "the local node is not a worker of this plan");
  ctx.local = lw;
  for (size_t i = 0; i < P.bufs.size(); ++i) {
    const PlanBuf& pb = P.bufs[i];
    northup_buf_s* ub = pb.kind == B_USER_A ? a : pb.kind == B_USER_B ? b : pb.kind == B_USER_C ? c : nullptr;
    if (ub) {
      ctx.base[i] = static_cast<char*>(ub->ptr);
      if (ub->storage == NU_FILE) ctx.file[i] = ub;
      continue;
    }
    if (pb.kind == B_REPLICA) {   // a sibling's replica of C (peer memory; same process)
      ctx.base[i] = static_cast<char*>(t->nodes[pb.node].replica);
      if (!ctx.base[i]) return fail(NU_ESTATE, "replica of node %d was unregistered", pb.node);
      continue;
    }
    if (lw >= 0 && pb.worker != lw) {   // a sibling's arena (IPC-mapped, pulls only)
      ctx.base[i] = pb.worker >= 0 && pb.worker < static_cast<int>(t->peers.size())
                        ? t->peers[pb.worker].arena : nullptr;
      continue;
    }
    int rc = ensure_arena(t, pb.node, pb.bytes);
    if (rc) return rc;
    ctx.base[i] = static_cast<char*>(t->nodes[pb.node].arena);
  }
  // Only record an event where some later op on another stream waits for it.
  std::vector<char> needs(P.ops.size(), 0);
  bool has_io = false, cross = false;
  for (const northup_op& op : P.ops) {
    for (int d = 0; d < op.ndeps; ++d) {
      needs[op.deps[d]] = 1;
      cross |= P.ops[op.deps[d]].worker != op.worker && !is_io_stream(P.ops[op.deps[d]].stream) &&
               !is_io_stream(op.stream);
    }
    has_io |= is_io_stream(op.stream);
  }
  ctx.needs_event = &needs;
  ctx.cross = cross;
  std::vector<uint64_t> needs_remote(P.ops.size(), 0);
  ctx.needs_remote = &needs_remote;
  if (lw >= 0 && cross) {
    if (t->peer_key != peer_key_of(P.M, P.N, P.K, o) ||
        static_cast<int>(t->peers.size()) != P.num_workers)
      return fail(NU_ESTATE, "multi-process siblings: run northup_peer_export/import for this GEMM first");
    for (int q = 0; q < P.num_workers; ++q)
      if (q != lw && !t->peers[q].flags)
        return fail(NU_ESTATE, "multi-process siblings: worker %d was not imported", q);
    for (const northup_op& op : P.ops)
      for (int d = 0; d < op.ndeps; ++d)
        if (op.worker != lw && P.ops[op.deps[d]].worker == lw)
          needs_remote[op.deps[d]] |= uint64_t(1) << op.worker;
    ctx.gen = ++t->gen;
  }
  ctx.issued.assign(P.ops.size(), 0);
  if (ctx.timing) t->timeline.clear();
  ctx.io_done.assign(P.ops.size(), 0);

  const int W = P.num_workers;
  // CUDA-graph mode: replay the captured op lists of an identical earlier call
  // (per-worker graphs cannot hold another worker's events: no graphs with
  // shared staging)
  const bool use_graph = o && o->graph && !has_io && !cross && !ctx.timing && lw < 0;
  std::vector<int64_t> key;
  if (use_graph) {
    key = graph_key(P, ctx.base, o);
    if (key == t->graph_key && static_cast<int>(t->graph_execs.size()) == W) {
      for (int wi = 0; wi < W; ++wi) {
        WorkerState* w = worker_for_node(t, P.worker_node[wi]);
        cudaSetDevice(w->device);
        cudaError_t e = cudaGraphLaunch(static_cast<cudaGraphExec_t>(t->graph_execs[wi]), w->streams[0]);
        if (e != cudaSuccess) return cuda_fail(e, "cudaGraphLaunch");
      }
      for (int wi = 0; wi < W; ++wi) {
        WorkerState* w = worker_for_node(t, P.worker_node[wi]);
        cudaSetDevice(w->device);
        cudaError_t e = cudaStreamSynchronize(w->streams[0]);
        if (e != cudaSuccess) return cuda_fail(e, "graph synchronize");
      }
      if (st) st->graph_replayed = 1;
      return 0;
    }
    destroy_graphs(t);
    t->graph_execs.assign(W, nullptr);
  }
  std::vector<int> rcs(W + 2, 0);        // workers, then the read and the write I/O threads
  std::vector<std::string> errs(W + 2);
  std::vector<std::vector<double>> busy(W, std::vector<double>(S_NUM, 0.0));
  auto worker_body = [&](int wi) {
    bind_worker_thread(t, P.worker_node[wi]);
    cudaGraphExec_t ge = nullptr;
    rcs[wi] = run_worker(ctx, wi, busy[wi].data(), use_graph ? &ge : nullptr);
    if (use_graph) t->graph_execs[wi] = ge;
    if (rcs[wi]) {
      errs[wi] = northup_last_error();
      ctx.abort = true;
      ctx.cv.notify_all();
    }
  };
  auto io_body = [&](int k) {
    rcs[W + k] = run_io(ctx, k == 0 ? S_IO : S_IOW);
    if (rcs[W + k]) {
      errs[W + k] = northup_last_error();
      ctx.abort = true;
      ctx.cv.notify_all();
    }
  };
  std::vector<int> mine;
  for (int wi = 0; wi < W; ++wi)
    if (lw < 0 || wi == lw) mine.push_back(wi);
  if (mine.size() == 1 && !has_io) {
    worker_body(mine[0]);
  } else {
    std::vector<std::thread> th;
    for (int wi : mine) th.emplace_back(worker_body, wi);
    if (has_io) {
      th.emplace_back(io_body, 0);
      th.emplace_back(io_body, 1);
    }
    for (auto& x : th) x.join();
  }
  // report the root cause first: an I/O thread's error (the workers then only
  // see "aborted: file I/O failed")
  for (int k : {W, W + 1})
    if (rcs[k]) {
      if (use_graph) destroy_graphs(t);
      return fail(rcs[k], "I/O thread %d: %s", k - W, errs[k].c_str());
    }
  for (int wi = 0; wi <= W + 1; ++wi)
    if (rcs[wi]) {
      if (use_graph) destroy_graphs(t);
      return fail(rcs[wi], "%s %d: %s", wi < W ? "worker" : "I/O thread", wi, errs[wi].c_str());
    }
  if (use_graph) t->graph_key = key;
  if (st) {
    for (int wi = 0; wi < W; ++wi) {
      st->t_h2d_ms += busy[wi][S_H2D];
      st->t_compute_ms += busy[wi][S_COMP];
      st->t_d2h_ms += busy[wi][S_D2H];
      st->t_p2p_ms += busy[wi][S_D2D];
    }
    st->t_io_ms = ctx.io_ms;
    st->file_direct_mode = ctx.io_mode;
  }
  return 0;
}

// ------------------------------------------------- NU_SCHED_QUEUE (NEXT-2)
// One host thread per HBM sibling.  A thread pops a C tile from the tail of
// its own queue (or, when that is empty, steals from the head of the longest
// other queue), appends the tile's ops to its private op list through
// its own rectangle tracker (so dependencies on its earlier tiles — panel
// slots, the two C-tile buffers — are exact) and issues them on its streams.
// A thread keeps at most two tiles in flight: before popping it waits for the
// tile before the previous one, so a slower sibling pops fewer tiles.
// NORTHUP_DEBUG_SLOW_SIBLING="w,pct" holds sibling w's compute stream for pct %
// of each leaf's nominal time before launching it, in every schedule (a test
// hook that emulates an asymmetric tree, Fig. 2: a slower GPU).
int execute_queue(northup_tree_s* t, int64_t M, int64_t N, int64_t K, northup_buf_s* a, northup_buf_s* b,
                  northup_buf_s* c, const northup_gemm_opts* o, northup_stats* st) {
  std::vector<int> hbm;
  for (int ch : t->nodes[0].children) hbm.push_back(ch);
  const int G = static_cast<int>(hbm.size());
  const int64_t kc = (o && o->k_chunk > 0) ? o->k_chunk : kDefaultKChunk;
  const int npass = o ? o->npass : 0;
  QueueShape q;
  int rc = choose_queue(t, hbm, M, N, K, kc, o ? o->queue_tiles : 0, &q);
  if (rc) return rc;
  for (int w = 0; w < G; ++w) {
    rc = ensure_arena(t, hbm[w], q.arena_bytes);
    if (rc) return rc;
  }
  std::vector<std::deque<int64_t>> queues;
  for (auto& v : queue_initial(G, q)) queues.emplace_back(v.begin(), v.end());
  std::mutex qm;
  int slow_pct = 0;
  const int slow_w = debug_slow_sibling(&slow_pct);
  std::vector<int> rcs(G, 0);
  std::vector<std::string> errs(G);
  std::vector<northup_stats> wst(G);
  std::vector<int64_t> stolen(G, 0), popped(G, 0);

  auto pop = [&](int w, bool* st_) -> int64_t {
    std::lock_guard<std::mutex> g(qm);
    if (!queues[w].empty()) {
      const int64_t x = queues[w].back();
      queues[w].pop_back();
      return x;
    }
    int v = -1;
    for (int u = 0; u < G; ++u)
      if (u != w && !queues[u].empty() && (v < 0 || queues[u].size() > queues[v].size())) v = u;
    if (v < 0) return -1;
    const int64_t x = queues[v].front();
    queues[v].pop_front();
    *st_ = true;
    return x;
  };

  auto body = [&](int w) -> int {
    WorkerState* ws = worker_for_node(t, hbm[w]);
    if (!ws) return fail(NU_ESTATE, "no worker state for node %d", hbm[w]);
    cudaError_t e = cudaSetDevice(ws->device);
    if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
    Plan Pw;
    Builder B;
    B.P = &Pw;
    const int bA = B.add_buf(B_USER_A, 0, -1, 0), bB = B.add_buf(B_USER_B, 0, -1, 0);
    const int bC = B.add_buf(B_USER_C, 0, -1, 0), bAr = B.add_buf(B_ARENA, hbm[w], 0, q.arena_bytes);
    char* base[4] = {static_cast<char*>(a->ptr), static_cast<char*>(b->ptr), static_cast<char*>(c->ptr),
                     static_cast<char*>(t->nodes[hbm[w]].arena)};
    std::vector<cudaEvent_t> evs;
    std::deque<cudaEvent_t> inflight;
    int64_t pctr = 0, ntask = 0;
    int result = 0;
    for (;;) {
      if (inflight.size() >= 2) {
        e = cudaEventSynchronize(inflight.front());
        if (e != cudaSuccess) { result = cuda_fail(e, "tile completion"); break; }
        inflight.pop_front();
      }
      bool was_stolen = false;
      const int64_t task = pop(w, &was_stolen);
      if (task < 0) break;
      popped[w]++;
      stolen[w] += was_stolen;
      const size_t first = Pw.ops.size();
      emit_task(B, 0, bAr, q, task, static_cast<int>(ntask & 1), &pctr, bA, bB, bC, M, N, K, &wst[w]);
      ++ntask;
      if (B.overflow) { result = fail(NU_ENOTSUP, "dependency fan-in above 16"); break; }
      for (size_t i = first; i < Pw.ops.size() && !result; ++i) {
        const northup_op& op = Pw.ops[i];
        cudaStream_t s = ws->streams[op.stream];
        for (int d = 0; d < op.ndeps; ++d) cudaStreamWaitEvent(s, evs[op.deps[d]], 0);
        if (op.op == NU_OP_COPY) {
          e = cudaMemcpy2DAsync(base[op.dst_buf] + op.dst_off * 4, op.dst_ld * 4, base[op.src_buf] + op.src_off * 4,
                                op.src_ld * 4, op.cols * 4, op.rows, cudaMemcpyDefault, s);
          if (e != cudaSuccess) result = cuda_fail(e, "copy");
        } else {
          if (w == slow_w && slow_pct > 0) debug_spin(debug_slow_ns(slow_pct, op.m, op.n, op.k), s);
          LeafCall lc{};
          lc.A = reinterpret_cast<const float*>(base[op.a_buf] + op.a_off * 4), lc.lda = op.lda;
          lc.B = reinterpret_cast<const float*>(base[op.b_buf] + op.b_off * 4), lc.ldb = op.ldb;
          lc.C = reinterpret_cast<float*>(base[op.c_buf] + op.c_off * 4), lc.ldc = op.ldc;
          lc.M = op.m, lc.N = op.n, lc.K = op.k, lc.accumulate = op.accumulate, lc.panel = kc, lc.npass = npass;
          lc.scratch = base[3] + (q.arena_bytes - q.scratch_bytes), lc.scratch_bytes = q.scratch_bytes;
          lc.stream = s;
          result = leaf_run(lc);
        }
        cudaEvent_t ev;
        e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventRecord(ev, s);
        if (e != cudaSuccess && !result) result = cuda_fail(e, "event");
        evs.push_back(ev);
      }
      if (result) break;
      inflight.push_back(evs.back());   // the tile's drain (D2H) is its last op
    }
    for (cudaStream_t s : ws->streams) {
      e = cudaStreamSynchronize(s);
      if (e != cudaSuccess && !result) result = cuda_fail(e, "stream synchronize");
    }
    for (cudaEvent_t ev : evs) cudaEventDestroy(ev);
    return result;
  };
  std::vector<std::thread> th;
  for (int w = 0; w < G; ++w)
    th.emplace_back([&, w] {
      bind_worker_thread(t, hbm[w]);
      rcs[w] = body(w);
      if (rcs[w]) errs[w] = northup_last_error();
    });
  for (auto& x : th) x.join();
  for (int w = 0; w < G; ++w)
    if (rcs[w]) return fail(rcs[w], "queue worker %d: %s", w, errs[w].c_str());
  st->bytes_h2d = st->bytes_d2h = 0;
  st->leaf_launches = 0;
  for (int w = 0; w < G; ++w) {
    st->bytes_h2d += wst[w].bytes_h2d;
    st->bytes_d2h += wst[w].bytes_d2h;
    st->leaf_launches += wst[w].leaf_launches;   // one launch per leaf op (bk = k_chunk)
    st->tasks_stolen += stolen[w];
  }
  st->tasks = q.Tr * q.Tc;
  return 0;
}

}  // namespace nu

// Debug (not in northup.h): per-op timeline of the last collect_timing run,
// rows of (op index, worker, stream, start ms, end ms).  Returns the row count.
extern "C" int northup_debug_timeline(northup_tree_t t, float* out, int cap_rows) {
  if (!t) return -1;
  const int n = static_cast<int>(t->timeline.size());
  for (int i = 0; i < n && i < cap_rows; ++i)
    for (int j = 0; j < 5; ++j) out[5 * i + j] = t->timeline[i][j];
  return n;
}
