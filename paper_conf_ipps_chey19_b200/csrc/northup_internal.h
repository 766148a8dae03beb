// Internal declarations shared by the translation units of libnorthup.so.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>
#include <sys/types.h>

#include <array>
#include <string>
#include <vector>

#include "northup.h"

namespace nu {

constexpr int kMaxDevices = 64;
constexpr int64_t kDefaultKChunk = 2048;   // K panel of one leaf launch / split (R20, R22)
constexpr int64_t kAccChunk = 256;         // TMEM accumulation length inside a panel (R20)
constexpr int kDefaultNpass = 3;            // 3 = fp16 hi.hi + hi.lo + lo.hi on the scaled split (R22)
constexpr int kSlots = 3;                  // staging ring depth per operand (reading R8)
constexpr int kRasterBand = 16;            // n-blocks per raster band in the leaf
constexpr int64_t kPanelChunks = 1;        // leaf K-panel launches, in k_chunks (0 = one launch)
constexpr int kHotspotMaxIters = 8;        // HotSpot-2D iterations per leaf launch (shared-memory border)

// Kernel launches issued by the library (all devices, all threads): the
// bench's `gpu_launches` claim (northup_debug_kernel_launches).
int sms_of(int dev);   // SM count of a device (cached)
void count_launches(int n);

// Positional file I/O for every FILE path (tree.cpp): pread / pwrite, unless a
// test armed a fault with NORTHUP_IO_FAULT="<read|write>:<eio|enospc|short|eof>:<n>"
// (the n-th call of that kind fails with EIO / ENOSPC, moves half the bytes, or
// returns 0).  The errno of the last failed I/O is kept (northup_last_io_errno).
ssize_t pio(int fd, void* p, size_t n, uint64_t off, bool write);
void note_io_errno(int e);

// Thread-local error message (northup_last_error).  Returns its argument so
// call sites can write `return fail(NU_EINVAL, "...")`.
void set_error(const char* fmt, ...) __attribute__((format(printf, 1, 2)));
int fail(int code, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
int cuda_fail(cudaError_t e, const char* what);

// ------------------------------------------------------------------ tree
struct Node {
  int id = -1;
  int storage = NU_HOST;
  int phys = -1;
  int processor = NU_PROC_NONE;
  uint64_t capacity = 0;    // bytes, 0 = unbounded
  uint64_t used = 0;        // bytes allocated by the library at this node
  int level = 0;
  int parent = -1;
  std::vector<int> children;
  int64_t bm = 0, bn = 0, bk = 0;   // block override (set_block)
  // HBM nodes: arena used for plan buffers (slots, C block, tail buffers).
  void* arena = nullptr;
  uint64_t arena_bytes = 0;
  bool arena_owned = false;
  // replicate_result target (caller-owned device buffer of M x N floats)
  void* replica = nullptr;
  uint64_t replica_bytes = 0;
};

}  // namespace nu

struct northup_buf_s {
  northup_tree_t tree = nullptr;
  int node = -1;
  int storage = NU_HOST;
  void* ptr = nullptr;       // host / device pointer (NULL for files)
  int fd = -1;               // file descriptor (NU_FILE)
  int direct_fd = -1;        // O_DIRECT descriptor when the file system allows it
  uint64_t bytes = 0;
  bool owned = false;        // library allocated (freed on release/destroy)
  bool registered = false;   // cudaHostRegister'ed by us (wrap_host)
  bool direct = false;       // fd opened with O_DIRECT
  std::string path;
};

struct WorkerState;

struct northup_tree_s {
  std::vector<nu::Node> nodes;
  bool finalized = false;
  bool busy = false;
  std::string file_dir = "/tmp";
  std::vector<northup_buf_s*> bufs;
  std::vector<WorkerState*> workers;   // one per HBM node (created at finalize)
  std::vector<void*> nccl_comms;       // ncclComm_t per HBM sibling (replicate_result)
  std::vector<std::array<float, 5>> timeline;   // last collect_timing run (debug)
  std::vector<void*> graph_execs;      // cudaGraphExec_t per worker (opts->graph)
  std::vector<int64_t> graph_key;      // the GEMM they were captured for
  // Multi-process siblings (northup_tree_set_local, peer.cpp): this process
  // runs only HBM node `local_node`; the other siblings' arenas and flag words
  // are mapped through CUDA IPC.  Cross-sibling dependencies become device-side
  // waits on the producer's flag word (cuStreamWaitValue32 >= gen), written
  // by the producer after the op (cuStreamWriteValue32).
  int local_node = -1;
  struct Peer {
    char* arena = nullptr;       // IPC-mapped arena of that sibling
    uint32_t* flags = nullptr;   // IPC-mapped flag words of that sibling
  };
  std::vector<Peer> peers;             // per plan worker
  uint32_t* flags = nullptr;           // this process's flag words: [w] = done of sibling w, [G + op]
  uint64_t flags_cap = 0;              // words
  std::vector<void*> flag_graveyard;   // outgrown flag buffers (peers may still map them)
  uint32_t gen = 0;                    // generation of the current call (monotonic)
  std::vector<int64_t> peer_key;       // the GEMM the peers were exported/imported for
  // Set at finalize (exec.cpp): every pair of distinct HBM devices has NVLink/P2P
  // access (else shared staging is not planned), the per-GPU PCIe bandwidth
  // measured with every local link busy in both directions (0 = not measured:
  // the planner's nominal constant), and the CPUs of each worker's NUMA node.
  bool p2p_ok = true;
  double pcie_gbs = 0.0;
  std::vector<std::vector<int>> worker_cpus;   // per HBM node id (empty: no binding)
};

namespace nu {

// --------------------------------------------------------------- plan
// S_NUM CUDA streams per worker (S_IO's slot unused); S_IO / S_IOW are the
// file-read and file-write queues of the I/O pseudo-worker (one host thread each)
enum Stream { S_H2D = 0, S_COMP = 1, S_D2H = 2, S_IO = 3, S_D2D = 4, S_NUM = 5, S_IOW = 5, S_KEYS = 6 };
inline bool is_io_stream(int s) { return s == S_IO || s == S_IOW; }
// B_REPLICA: the caller's M x N replica of C at an HBM node (replicate_result, pushed
// region by region as the drains run: see Builder::push_replicas)
enum BufKind { B_USER_A = 0, B_USER_B = 1, B_USER_C = 2, B_ARENA = 3, B_DRAM = 4, B_REPLICA = 5 };

struct PlanBuf {
  int kind = B_ARENA;
  int node = -1;
  int worker = -1;
  uint64_t bytes = 0;   // elements * 4 for arenas (planned footprint)
};

struct Plan {
  int64_t M = 0, N = 0, K = 0;
  int num_workers = 0;
  std::vector<int> worker_node;      // HBM node id per worker
  std::vector<PlanBuf> bufs;
  std::vector<northup_op> ops;
  northup_stats stats{};
  int64_t kc = kDefaultKChunk;
  int npass = 3;
  bool root_is_device = false;
  bool file_root = false;
  bool replica_push = false;          // replicate_result is carried by the plan's own copies
  // Leaf scratch per worker (split operands of one K panel, leaf_scratch_bytes):
  // the last `scr_bytes` of arena buffer `scr_buf`, at byte offset `scr_off`.
  std::vector<int> scr_buf;
  std::vector<uint64_t> scr_off, scr_bytes;
  float hs_coef[5] = {};                // HotSpot-2D plans: cap_1, rx_1, ry_1, rz_1, amb
};

int build_plan(const northup_tree_s* t, int64_t M, int64_t N, int64_t K,
               const northup_gemm_opts* o, Plan* out);
int execute_queue(northup_tree_s* t, int64_t M, int64_t N, int64_t K, northup_buf_s* a,
                  northup_buf_s* b, northup_buf_s* c, const northup_gemm_opts* o, northup_stats* st);
// a_aligned / b_aligned: the root-tier device pointers are 16-B aligned
// (only consulted for an HBM root, where the leaf reads them in place).
int build_plan_ex(const northup_tree_s* t, int64_t M, int64_t N, int64_t K,
                  const northup_gemm_opts* o, bool a_aligned, bool b_aligned, Plan* out);
int partition_grid(int G, int64_t M, int64_t N, int* Pr, int* Pc);

// NU_SCHED_QUEUE (S§8(f) NEXT-2): C tiles in per-sibling work queues.
struct QueueShape {
  int64_t tm = 0, tn = 0, bk = 0;   // tile rows / cols, K panel
  int64_t Tr = 0, Tc = 0;           // tile grid
  uint64_t arena_bytes = 0;         // per sibling: 2 C-tile buffers + kSlots panel slots + leaf scratch
  uint64_t scratch_bytes = 0;       // the leaf scratch at the end of that arena
};
int choose_queue(const northup_tree_s* t, const std::vector<int>& hbm, int64_t M, int64_t N,
                 int64_t K, int64_t kc, int tiles, QueueShape* q);
// Initial queues: tiles in row-major order, contiguous chunks per sibling.
std::vector<std::vector<int64_t>> queue_initial(int G, const QueueShape& q);
struct Builder;
// Append the ops of tile `task` for sibling w (arena buffer `arena`, C-tile
// buffer `cslot` of 2, panel-slot counter `pctr`) to B.
void emit_task(Builder& B, int w, int arena, const QueueShape& q, int64_t task, int cslot,
               int64_t* pctr, int A, int Bb, int C, int64_t M, int64_t N, int64_t K, northup_stats* st);
int region_of(int G, int64_t M, int64_t N, int r, int64_t* r0, int64_t* r1, int64_t* c0,
              int64_t* c1);
int validate_tree(const northup_tree_s* t);

// --------------------------------------------------------------- leaf
// One leaf call (leaf_host.cu): C (+)= A.B over K, one split + GEMM per K panel.
struct LeafCall {
  const float* A;
  int64_t lda;
  const float* B;          // raw fp32 (eb_presplit == NULL) or split in place (split.cu layout)
  int64_t ldb;
  const int* eb_presplit;  // B's column exponents, [panel p][eb_stride]
  int64_t eb_stride;
  float* C;
  int64_t ldc;
  int64_t M, N, K;
  int accumulate;
  int64_t panel;           // K per launch (0 = kDefaultKChunk)
  int npass;
  char* scratch;           // NULL: stream-ordered from the leaf's pool
  uint64_t scratch_bytes;
  float* dbg;
  cudaStream_t stream;
  // Debug timing: events recorded around each GEMM kernel (2 per launch, up
  // to n_events) on `stream`; *events_used returns how many were recorded.
  cudaEvent_t* events = nullptr;
  int n_events = 0;
  int* events_used = nullptr;
};
int leaf_run(const LeafCall& c);
namespace leaf {
// In-place or out-of-place split of a B panel (split.cu); bmax: N words of scratch.
int split_b_launch(const float* B, int64_t ldb, int Kl, int N, float* dst, int64_t ldd, int* eb,
                   unsigned* bmax, cudaStream_t s);
}  // namespace leaf
uint64_t leaf_scratch_bytes(int64_t m, int64_t n, int64_t panel, bool b_presplit);
// Scratch of the largest leaf op over an m x n C block (256-B rounded).
inline uint64_t leaf_scratch(int64_t m, int64_t n, int64_t panel) {
  return (leaf_scratch_bytes(m, n, panel, false) + 255) / 256 * 256;
}
constexpr int64_t kLeafMaxN = 32768;   // columns of B split at a time (leaf_run)
int64_t leaf_acc_chunk();
bool leaf_tma_legal(const void* p, int64_t ld);
int leaf_gemm_launch(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                     int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t kc,
                     int npass, cudaStream_t stream);

// --------------------------------------------------------------- HotSpot-2D
// The leaf (hotspot.cu): `iters` (<= kHotspotMaxIters) iterations on a window
// wm x wn at grid origin (gy0, gx0) of an R x C grid; writes the window's valid
// region (shrunk by `iters` on every side that is not a grid edge) into tout,
// which has the window's shape.
int hotspot_launch(const float* tin, int64_t ldt, const float* pw, int64_t ldp, float* tout,
                   int64_t ldo, int64_t wm, int64_t wn, int64_t gy0, int64_t gx0, int64_t R,
                   int64_t C, int iters, const float coef[5], cudaStream_t stream);
int build_hotspot_plan(const northup_tree_s* t, int64_t R, int64_t C, int64_t iters,
                       const northup_hotspot_opts* o, const northup_hotspot_coeffs* k, Plan* out);

// Test hooks: a kernel that holds a stream for `ns` ns; the sibling (and the
// slowdown in percent) named by NORTHUP_DEBUG_SLOW_SIBLING="w,pct" (-1 = none).
// The executors hold that sibling's compute stream for pct % of each leaf's
// nominal time (2mnk at 300 TF/s) before launching it: a slower GPU.
int debug_spin(long long ns, cudaStream_t s);
// Force-load the kernels (lazy module loading) on the current device; hotspot.cu's part.
void preload_kernels();
// One-thread kernel: system-scope release store of v to addr (multi-process flag words).
int flag_store_launch(uint32_t* addr, uint32_t v, cudaStream_t s);
void hotspot_preload();
int debug_slow_sibling(int* pct);
inline long long debug_slow_ns(int pct, int64_t m, int64_t n, int64_t k) {
  return static_cast<long long>(pct / 100.0 * 2.0 * m * n * k / 3e14 * 1e9);
}

// --------------------------------------------------------------- executor
int execute_plan(northup_tree_s* t, const Plan& plan, northup_buf_s* a, northup_buf_s* b,
                 northup_buf_s* c, const northup_gemm_opts* o, northup_stats* st);
int finalize_workers(northup_tree_s* t);
void numa_bind_plan(northup_tree_s* t);
void bind_worker_thread(const northup_tree_s* t, int node);
int calibrate_pcie(northup_tree_s* t);
int ensure_arena(northup_tree_s* t, int node, uint64_t bytes);
// Multi-process siblings (peer.cpp)
std::vector<int64_t> peer_key_of(int64_t M, int64_t N, int64_t K, const northup_gemm_opts* o);
int local_worker(const northup_tree_s* t, const Plan& P);   // -1 when every worker is local
int stream_wait_flag(cudaStream_t s, const uint32_t* addr, uint32_t gen);
int stream_write_flag(cudaStream_t s, uint32_t* addr, uint32_t gen);
void destroy_peers(northup_tree_s* t);
int gather_replicas(northup_tree_s* t, const Plan& P, northup_buf_s* C, northup_stats* st);
void destroy_nccl(northup_tree_s* t);
void destroy_graphs(northup_tree_s* t);
void destroy_workers(northup_tree_s* t);

}  // namespace nu

struct northup_plan_s {
  nu::Plan plan;
};
