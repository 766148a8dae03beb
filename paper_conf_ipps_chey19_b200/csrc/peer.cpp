// Multi-process siblings: one process per GPU (the S§8(e) process model under
// torchrun), each running one HBM sibling of the same tree, with the
// shared-staging pulls of NEXT-1 (P:230 siblings; P:409 streaming over
// networks) going straight to the peers' HBM.
//
//   northup_tree_set_local(t, node)   this process runs HBM node `node` only
//   northup_peer_export(t, M, N, K)   plan the GEMM, allocate the local arena
//                                     and flag words, return CUDA IPC handles
//   northup_peer_import(t, w, blob)   map sibling w's arena and flag words
//
// Every process builds the same plan (same tree, sizes and options), so op
// indices agree.  Each process owns G + nops flag words in its own HBM:
// [w] = sibling w's done word, [G + i] = op i.  A dependency of a local op on a
// sibling's op i is a device-side wait on the LOCAL word
// `cuStreamWaitValue32(flags[G + i] >= gen)`; after op i the producing sibling
// stores `gen` into the flag words of every process that waits for it through
// the IPC-mapped peer address (a one-thread kernel: __threadfence_system, then a
// system-scope release store, so the op's data is visible first).  Consumers
// only poll local memory.
// No host thread blocks on a peer: the waits form a DAG because every
// dependency points backwards in plan order and each stream is FIFO in plan
// order.  At the end of a call every process stores its done word into all
// siblings and waits for theirs (a device-side join), so no sibling can still
// be pulling from an arena when northup_gemm returns.
#include <stdlib.h>
#include <string.h>

#include "northup_internal.h"

namespace nu {

namespace {

using PFN_wait32 = int (*)(cudaStream_t, unsigned long long, unsigned int, unsigned int);
PFN_wait32 g_wait = nullptr;
constexpr unsigned kWaitGeq = 0x0;        // CU_STREAM_WAIT_VALUE_GEQ
constexpr uint32_t kMagic = 0x4e555052;   // "NUPR"

int load_mem_ops() {
  if (g_wait) return 0;
  void* fw = nullptr;
  cudaDriverEntryPointQueryResult q1;
  cudaError_t e1 = cudaGetDriverEntryPointByVersion("cuStreamWaitValue32", &fw, 12000, cudaEnableDefault, &q1);
  if (e1 != cudaSuccess || q1 != cudaDriverEntryPointSuccess || !fw)
    return fail(NU_ECUDA, "stream memory operations (cuStreamWaitValue32) unavailable");
  g_wait = reinterpret_cast<PFN_wait32>(fw);
  return 0;
}

struct Blob {
  uint32_t magic;
  int32_t worker;
  int64_t M, N, K;
  uint64_t nops;
  uint64_t arena_bytes;
  int64_t key_hash;
  cudaIpcMemHandle_t arena;
  cudaIpcMemHandle_t flags;
};

int64_t hash_key(const std::vector<int64_t>& k) {
  uint64_t h = 1469598103934665603ull;
  for (int64_t v : k) h = (h ^ static_cast<uint64_t>(v)) * 1099511628211ull;
  return static_cast<int64_t>(h);
}

}  // namespace

std::vector<int64_t> peer_key_of(int64_t M, int64_t N, int64_t K, const northup_gemm_opts* o) {
  return {M, N, K, o ? o->schedule : 0, o ? o->k_chunk : 0, o ? o->shared_staging : 0};
}

int local_worker(const northup_tree_s* t, const Plan& P) {
  if (t->local_node < 0) return -1;
  for (int w = 0; w < P.num_workers; ++w)
    if (P.worker_node[w] == t->local_node) return w;
  return -2;
}

int stream_wait_flag(cudaStream_t s, const uint32_t* addr, uint32_t gen) {
  int rc = load_mem_ops();
  if (rc) return rc;
  int r = g_wait(s, reinterpret_cast<unsigned long long>(addr), gen, kWaitGeq);
  return r ? fail(NU_ECUDA, "cuStreamWaitValue32 failed (%d)", r) : 0;
}

int stream_write_flag(cudaStream_t s, uint32_t* addr, uint32_t gen) {
  // the store into a sibling's flag word: a one-thread kernel with a release store
  // at system scope (valid for any peer-mapped address, including another GPU's
  // memory over NVLink, where a stream memory operation is not guaranteed to be)
  return flag_store_launch(addr, gen, s);
}

static void close_peer(northup_tree_s* t, int w) {
  if (w < 0 || w >= static_cast<int>(t->peers.size())) return;
  auto& p = t->peers[w];
  if (p.arena) cudaIpcCloseMemHandle(p.arena);
  if (p.flags) cudaIpcCloseMemHandle(p.flags);
  p.arena = nullptr;
  p.flags = nullptr;
}

void destroy_peers(northup_tree_s* t) {
  int dev = t->local_node >= 0 ? t->nodes[t->local_node].phys : -1;
  if (dev >= 0) cudaSetDevice(dev);
  for (int w = 0; w < static_cast<int>(t->peers.size()); ++w) close_peer(t, w);
  t->peers.clear();
  if (t->flags) cudaFree(t->flags);
  for (void* p : t->flag_graveyard) cudaFree(p);
  t->flags = nullptr;
  t->flag_graveyard.clear();
  t->flags_cap = 0;
}

}  // namespace nu

using namespace nu;

extern "C" {

int northup_peer_export(northup_tree_t t, int64_t M, int64_t N, int64_t K, const northup_gemm_opts* o,
                        void* blob, uint64_t cap, uint64_t* len) {
  if (!t || !len) return fail(NU_EINVAL, "NULL argument");
  *len = sizeof(Blob);
  if (!blob || cap < sizeof(Blob)) return fail(NU_EINVAL, "blob needs %zu bytes", sizeof(Blob));
  if (!t->finalized) return fail(NU_ESTATE, "tree not finalized");
  if (t->local_node < 0) return fail(NU_ESTATE, "northup_tree_set_local was not called");
  if (t->busy) return fail(NU_ESTATE, "a northup_gemm is in flight on this tree");
  Plan P;
  int rc = build_plan(t, M, N, K, o, &P);
  if (rc) return rc;
  const int lw = local_worker(t, P);
  if (lw < 0) return fail(NU_ESTATE, "the local node is not a worker of this plan");
  if (P.num_workers > 64) return fail(NU_ENOTSUP, "multi-process siblings support at most 64 GPUs");
  const Node& ln = t->nodes[t->local_node];
  cudaError_t e = cudaSetDevice(ln.phys);
  if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
  for (const PlanBuf& pb : P.bufs)
    if (pb.kind == B_ARENA && pb.node == t->local_node) {
      rc = ensure_arena(t, pb.node, pb.bytes);
      if (rc) return rc;
    }
  if (!ln.arena) {   // no work for this sibling (tiny problem): export a 256-B arena
    rc = ensure_arena(t, t->local_node, 256);
    if (rc) return rc;
  }
  if (!t->nodes[t->local_node].arena_owned)
    return fail(NU_ENOTSUP, "peer export needs a library-owned arena (not northup_tree_set_arena)");
  const uint64_t words = P.ops.size() + P.num_workers;
  if (words > t->flags_cap) {
    // Outgrown flag buffers stay allocated until destroy: a slower sibling may
    // still wait on them (waits are GEQ on a monotonic generation).
    if (t->flags) t->flag_graveyard.push_back(t->flags);
    t->flags = nullptr;
    const uint64_t cap_words = std::max<uint64_t>(words, 1 << 16);
    e = cudaMalloc(&t->flags, cap_words * 4);
    if (e == cudaSuccess) e = cudaMemset(t->flags, 0, cap_words * 4);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_fail(e, "flag words");
    t->flags_cap = cap_words;
    // a fresh buffer restarts the generations every sibling waits for
    t->gen = 0;
  }
  Blob b{};
  b.magic = kMagic;
  b.worker = lw;
  b.M = M;
  b.N = N;
  b.K = K;
  b.nops = P.ops.size();
  b.arena_bytes = t->nodes[t->local_node].arena_bytes;
  t->peer_key = peer_key_of(M, N, K, o);
  b.key_hash = hash_key(t->peer_key);
  e = cudaIpcGetMemHandle(&b.arena, t->nodes[t->local_node].arena);
  if (e != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle(arena)");
  e = cudaIpcGetMemHandle(&b.flags, t->flags);
  if (e != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle(flags)");
  memcpy(blob, &b, sizeof(b));
  t->peers.assign(P.num_workers, northup_tree_s::Peer{});
  return 0;
}

int northup_peer_import(northup_tree_t t, int worker, const void* blob, uint64_t len) {
  if (!t || !blob) return fail(NU_EINVAL, "NULL argument");
  if (len < sizeof(Blob)) return fail(NU_EINVAL, "blob too short");
  if (t->local_node < 0) return fail(NU_ESTATE, "northup_tree_set_local was not called");
  Blob b;
  memcpy(&b, blob, sizeof(b));
  if (b.magic != kMagic) return fail(NU_EINVAL, "not a northup peer blob");
  if (t->peer_key.empty() || b.key_hash != hash_key(t->peer_key))
    return fail(NU_ESTATE, "peer blob is for another GEMM; export this one first");
  if (worker != b.worker || worker < 0 || worker >= static_cast<int>(t->peers.size()))
    return fail(NU_EINVAL, "blob belongs to worker %d, not %d", b.worker, worker);
  cudaError_t e = cudaSetDevice(t->nodes[t->local_node].phys);
  if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
  close_peer(t, worker);
  void* a = nullptr;
  void* f = nullptr;
  e = cudaIpcOpenMemHandle(&a, b.arena, cudaIpcMemLazyEnablePeerAccess);
  if (e == cudaErrorInvalidDevice || e == cudaErrorInvalidResourceHandle) {
    // the sibling is this very process (handles cannot be opened by their
    // owner): nothing to map
    cudaGetLastError();
    return fail(NU_EINVAL, "cannot import a blob exported by this process");
  }
  if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle(arena)");
  e = cudaIpcOpenMemHandle(&f, b.flags, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    cudaIpcCloseMemHandle(a);
    return cuda_fail(e, "cudaIpcOpenMemHandle(flags)");
  }
  t->peers[worker].arena = static_cast<char*>(a);
  t->peers[worker].flags = static_cast<uint32_t*>(f);
  return 0;
}

}  // extern "C"
