// Optional final gather (S§8(e), `replicate_result`): after the join every
// GPU holds the whole C (M x N) in a caller-registered HBM replica buffer.
//
// Each sibling first places its own C region into its replica (from the
// resident HBM C block when the plan kept the whole region there, else from
// the root tier over PCIe), then the regions are exchanged over NVLink:
//   * distinct devices: NCCL (loaded with dlopen, so the library has no link
//     dependency and shares the process's NCCL when PyTorch already loaded
//     one) — one ncclBroadcast per region inside a group; row-strip regions
//     (Pc = 1) broadcast straight into place, 2-D regions one at a time
//     through a region-sized staging buffer (the idle arena, or a buffer
//     counted against the node's capacity);
//   * siblings aliasing one device ("virtual siblings", tests): device copies.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <mutex>
#include <vector>

#include "northup_internal.h"

namespace nu {

namespace {

struct NcclApi {
  bool ok = false;
  ncclResult_t (*CommInitAll)(ncclComm_t*, int, const int*) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    api.CommInitAll = reinterpret_cast<decltype(api.CommInitAll)>(dlsym(h, "ncclCommInitAll"));
    api.CommDestroy = reinterpret_cast<decltype(api.CommDestroy)>(dlsym(h, "ncclCommDestroy"));
    api.GroupStart = reinterpret_cast<decltype(api.GroupStart)>(dlsym(h, "ncclGroupStart"));
    api.GroupEnd = reinterpret_cast<decltype(api.GroupEnd)>(dlsym(h, "ncclGroupEnd"));
    api.Broadcast = reinterpret_cast<decltype(api.Broadcast)>(dlsym(h, "ncclBroadcast"));
    api.GetErrorString = reinterpret_cast<decltype(api.GetErrorString)>(dlsym(h, "ncclGetErrorString"));
    api.ok = api.CommInitAll && api.CommDestroy && api.GroupStart && api.GroupEnd && api.Broadcast &&
             api.GetErrorString;
  });
  return api;
}

int nccl_fail(ncclResult_t r, const char* what) {
  return fail(NU_ENCCL, "%s: %s", what, nccl().GetErrorString ? nccl().GetErrorString(r) : "?");
}

}  // namespace

void destroy_nccl(northup_tree_s* t) {
  for (void* c : t->nccl_comms)
    if (c && nccl().ok) nccl().CommDestroy(static_cast<ncclComm_t>(c));
  t->nccl_comms.clear();
}

int gather_replicas(northup_tree_s* t, const Plan& P, northup_buf_s* C, northup_stats* st) {
  const int G = P.num_workers;
  const int64_t M = P.M, N = P.N;
  std::vector<void*> rep(G, nullptr);
  std::vector<int> dev(G);
  for (int w = 0; w < G; ++w) {
    const Node& n = t->nodes[P.worker_node[w]];
    if (!n.replica || n.replica_bytes < static_cast<uint64_t>(M) * N * 4)
      return fail(NU_EINVAL, "replicate_result: HBM node %d has no M x N replica buffer "
                             "(northup_tree_set_replica)", n.id);
    rep[w] = n.replica;
    dev[w] = n.phys;
  }
  // 1. own region into own replica
  std::vector<int64_t> r0(G), r1(G), c0(G), c1(G);
  for (int w = 0; w < G; ++w) {
    int rc = region_of(G, M, N, w, &r0[w], &r1[w], &c0[w], &c1[w]);
    if (rc) return rc;
    const int64_t m = r1[w] - r0[w], n = c1[w] - c0[w];
    if (m <= 0 || n <= 0) continue;
    cudaSetDevice(dev[w]);
    const bool resident = P.stats.bm >= m && P.stats.bn >= n && !P.file_root && !P.root_is_device &&
                          P.stats.schedule == NU_SCHED_S2;
    const Node& hn = t->nodes[P.worker_node[w]];
    const char* src;
    int64_t ld;
    if (resident && hn.arena) {
      src = static_cast<const char*>(hn.arena);   // C block at arena offset 0 (plan.cpp S2 layout)
      ld = std::max<int64_t>(32, (n + 31) / 32 * 32);
    } else {
      src = static_cast<const char*>(C->ptr) + (r0[w] * N + c0[w]) * 4;
      ld = N;
    }
    cudaError_t e = cudaMemcpy2D(static_cast<char*>(rep[w]) + (r0[w] * N + c0[w]) * 4, N * 4, src,
                                 ld * 4, n * 4, m, cudaMemcpyDefault);
    if (e != cudaSuccess) return cuda_fail(e, "replica: own region");
    if (!resident) st->bytes_h2d += static_cast<uint64_t>(m) * n * 4;
  }
  if (G == 1) return 0;
  std::vector<int> sorted = dev;
  std::sort(sorted.begin(), sorted.end());
  const bool distinct = std::unique(sorted.begin(), sorted.end()) == sorted.end();
  int Pr = 1, Pc = 1;
  partition_grid(G, M, N, &Pr, &Pc);
  if (distinct && nccl().ok) {
    // 2a. NCCL over NVLink: one broadcast per region, all in one group.
    if (t->nccl_comms.size() != static_cast<size_t>(G)) {
      destroy_nccl(t);
      std::vector<ncclComm_t> comms(G);
      ncclResult_t r = nccl().CommInitAll(comms.data(), G, dev.data());
      if (r != ncclSuccess) return nccl_fail(r, "ncclCommInitAll");
      for (auto c : comms) t->nccl_comms.push_back(c);
    }
    if (Pc > 1) {
      // 2-D regions are not contiguous in the replica: broadcast one region at
      // a time through a region-sized staging buffer on every GPU.  The staging
      // is the node's arena (idle after the join) when it is large enough, else
      // a buffer counted in the node's `used` (capacity checked) and freed on
      // every path.
      int64_t maxe = 0;
      for (int w = 0; w < G; ++w) maxe = std::max(maxe, (r1[w] - r0[w]) * (c1[w] - c0[w]));
      const uint64_t need = static_cast<uint64_t>(maxe) * 4;
      struct Staging {
        northup_tree_s* t;
        std::vector<void*> own;     // buffers we allocated (not arenas)
        std::vector<int> node;
        ~Staging() {
          for (size_t w = 0; w < own.size(); ++w)
            if (own[w]) {
              cudaSetDevice(t->nodes[node[w]].phys);
              cudaFree(own[w]);
            }
        }
      } stage{t, std::vector<void*>(G, nullptr), std::vector<int>(P.worker_node.begin(), P.worker_node.end())};
      std::vector<char*> sbuf(G, nullptr);
      std::vector<uint64_t> counted(G, 0);
      struct UsedGuard {
        northup_tree_s* t;
        const std::vector<int>& node;
        std::vector<uint64_t>& counted;
        ~UsedGuard() {
          for (size_t w = 0; w < counted.size(); ++w) t->nodes[node[w]].used -= counted[w];
        }
      } used_guard{t, stage.node, counted};
      for (int w = 0; w < G; ++w) {
        Node& hn = t->nodes[P.worker_node[w]];
        if (hn.arena && hn.arena_bytes >= need) {
          sbuf[w] = static_cast<char*>(hn.arena);
          continue;
        }
        if (hn.capacity && hn.used + need > hn.capacity)
          return fail(NU_ENOMEM, "replicate_result: node %d needs %llu B of staging beyond its capacity", hn.id,
                      (unsigned long long)need);
        cudaSetDevice(dev[w]);
        cudaError_t e = cudaMalloc(&stage.own[w], need);
        if (e != cudaSuccess) return cuda_fail(e, "replica: staging buffer");
        sbuf[w] = static_cast<char*>(stage.own[w]);
        hn.used += need;
        counted[w] = need;
      }
      for (int root = 0; root < G; ++root) {
        const int64_t m = r1[root] - r0[root], n = c1[root] - c0[root];
        if (m <= 0 || n <= 0) continue;
        cudaSetDevice(dev[root]);
        cudaError_t e = cudaMemcpy2D(sbuf[root], n * 4, static_cast<char*>(rep[root]) + (r0[root] * N + c0[root]) * 4,
                                     N * 4, n * 4, m, cudaMemcpyDeviceToDevice);
        if (e != cudaSuccess) return cuda_fail(e, "replica: pack region");
        ncclResult_t r = nccl().GroupStart();
        if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
        for (int w = 0; w < G && r == ncclSuccess; ++w)
          r = nccl().Broadcast(sbuf[w], sbuf[w], static_cast<size_t>(m * n), ncclFloat32, root,
                               static_cast<ncclComm_t>(t->nccl_comms[w]), 0);
        ncclResult_t r2 = nccl().GroupEnd();
        if (r != ncclSuccess) return nccl_fail(r, "ncclBroadcast");
        if (r2 != ncclSuccess) return nccl_fail(r2, "ncclGroupEnd");
        for (int w = 0; w < G; ++w) {
          if (w == root) continue;
          cudaSetDevice(dev[w]);
          e = cudaMemcpy2DAsync(static_cast<char*>(rep[w]) + (r0[root] * N + c0[root]) * 4, N * 4, sbuf[w], n * 4,
                                n * 4, m, cudaMemcpyDeviceToDevice, 0);
          if (e != cudaSuccess) return cuda_fail(e, "replica: unpack region");
        }
        for (int w = 0; w < G; ++w) {   // the staging is reused by the next region
          cudaSetDevice(dev[w]);
          e = cudaDeviceSynchronize();
          if (e != cudaSuccess) return cuda_fail(e, "replica: region sync");
        }
      }
    } else {
      nccl().GroupStart();
      for (int root = 0; root < G; ++root)
        for (int w = 0; w < G; ++w) {
          char* buf = static_cast<char*>(rep[w]) + r0[root] * N * 4;
          ncclResult_t r = nccl().Broadcast(buf, buf, static_cast<size_t>((r1[root] - r0[root]) * N),
                                            ncclFloat32, root, static_cast<ncclComm_t>(t->nccl_comms[w]), 0);
          if (r != ncclSuccess) {
            nccl().GroupEnd();
            return nccl_fail(r, "ncclBroadcast");
          }
        }
      ncclResult_t r = nccl().GroupEnd();
      if (r != ncclSuccess) return nccl_fail(r, "ncclGroupEnd");
      for (int w = 0; w < G; ++w) {
        cudaSetDevice(dev[w]);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) return cuda_fail(e, "replica: broadcast sync");
      }
    }
  } else {
    // 2b. aliased devices (or no NCCL): device-to-device copies of each region
    for (int w = 0; w < G; ++w)
      for (int root = 0; root < G; ++root) {
        if (root == w) continue;
        const int64_t m = r1[root] - r0[root], n = c1[root] - c0[root];
        if (m <= 0 || n <= 0) continue;
        const size_t off = static_cast<size_t>(r0[root] * N + c0[root]) * 4;
        cudaError_t e = cudaMemcpy2D(static_cast<char*>(rep[w]) + off, N * 4,
                                     static_cast<char*>(rep[root]) + off, N * 4, n * 4, m,
                                     cudaMemcpyDefault);
        if (e != cudaSuccess) return cuda_fail(e, "replica: device copy");
      }
  }
  st->bytes_d2d += static_cast<uint64_t>(G - 1) * M * N * 4;
  return 0;
}

}  // namespace nu

extern "C" int northup_tree_set_replica(northup_tree_t t, int node, void* dev_ptr, uint64_t bytes) {
  using namespace nu;
  if (!t || node < 0 || node >= static_cast<int>(t->nodes.size()))
    return fail(NU_EINVAL, "unknown node %d", node);
  Node& n = t->nodes[node];
  if (n.storage != NU_HBM) return fail(NU_EINVAL, "replica buffers live at HBM nodes");
  n.replica = dev_ptr;
  n.replica_bytes = dev_ptr ? bytes : 0;
  return 0;
}
