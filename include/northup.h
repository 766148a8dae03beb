/*
 * northup.h — C ABI of the B200-native Northup out-of-core recursive GEMM.
 *
 * Northup (Che & Yin, PAPER.md) models a machine as a tree of memory nodes:
 * level 0 is the slowest storage, faster memories have larger levels, and a
 * leaf is the point where a processor computes (§III-B, Listing 1).  A
 * problem is split recursively; chunks move down a tree edge (`data_down`),
 * the child recurses, and results move back up (`data_up`) (Listing 3,
 * P:167-228).  This library implements the dense matrix-multiply case study
 * (§IV-A) on that tree:  root (pinned host DRAM, or a file with a
 * DRAM staging level) -> HBM of one or more B200s -> SMEM/TMEM leaf.
 *
 * Conventions (apply to every call unless stated):
 *   - Every function returns an int status: NU_OK (0) or a negative NU_E*.
 *     `northup_last_error()` returns a thread-local message for the last
 *     failure on the calling thread.
 *   - Matrices are fp32, dense, ROW-MAJOR (reading R1): A is M x K,
 *     B is K x N, C is M x N; leading dimensions are in elements.
 *   - Ownership: the caller owns the memory it wraps (A, B, C).  The tree owns
 *     every buffer it allocates (HBM slots, DRAM staging, files it creates)
 *     and frees them in northup_tree_destroy.  northup_buf_t handles belong to
 *     the tree that produced them.
 *   - A tree is not thread-safe; separate trees are independent.  Only one
 *     northup_gemm may be in flight per tree.  northup_gemm is synchronous.
 *   - Functions that only build or query the tree (create, add_node,
 *     set_block, queries, print, plan) never touch a GPU.
 */
#ifndef NORTHUP_H
#define NORTHUP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define NORTHUP_VERSION 100 /* 1.0.0 */

/* ------------------------------------------------------------ status codes */
#define NU_OK 0
#define NU_EINVAL (-1)  /* null/bad argument, bad dimensions, unknown node     */
#define NU_ENOMEM (-2)  /* capacity below the minimum block, or alloc failure  */
#define NU_EIO (-3)     /* file I/O failure (errno preserved)                  */
#define NU_ECUDA (-4)   /* CUDA runtime / driver failure                       */
#define NU_ENCCL (-5)   /* NCCL failure                                        */
#define NU_ESTATE (-6)  /* tree not finalized / already finalized / busy       */
#define NU_ENOTSUP (-7) /* valid but unsupported tree shape or option          */

/* ------------------------------------------- storage and processor types */
/* memory_t.storage_type of Listing 1. */
#define NU_FILE 0 /* file-backed storage (NVMe where present)   */
#define NU_HOST 1 /* host DRAM (pinned by the library)          */
#define NU_HBM 2  /* device memory of one B200 (physical_id = device ordinal) */
#define NU_SMEM 3 /* on-chip SMEM/TMEM of the leaf kernel       */

/* processor_t.processor_type of Listing 1, leaf only. */
#define NU_PROC_NONE 0
#define NU_PROC_SM100 1 /* B200 streaming multiprocessors (tcgen05 leaf kernel) */

/* Schedules for the HOST -> HBM edge (§IV-A). */
#define NU_SCHED_AUTO 0
#define NU_SCHED_S1 1 /* paper-literal: row shard m stays at l+1, column shards stream */
#define NU_SCHED_S2 2 /* C block resident, K panels stream, staggered C drain */
#define NU_SCHED_QUEUE 3 /* S§8(f) NEXT-2: C is cut into tiles held in one
                            work queue per HBM sibling; each sibling pops tiles from the tail of its
                            own queue and, when empty, steals from the head of another's; a tile is
                            an S2 sub-problem (C tile resident, K panels stream, tile drained).
                            HOST root, single process; no shared staging, no graphs. */
#define NU_SCHED_S2B 4 /* S2's B-first variant: all of B stays resident in HBM (split once,
                          in place, as its K panels land); rows [0, r1) of the C block are computed
                          while B streams in, the other rows then run as strips over the full K while
                          the first rows drain, so C's D2H overlaps compute instead of following it.
                          NU_SCHED_AUTO picks it over S2 when the cost model predicts a shorter block
                          time; NU_SCHED_S2 never uses it.  Not with NVLink-shared staging. */

typedef struct northup_tree_s* northup_tree_t;
typedef struct northup_buf_s* northup_buf_t;

/* Snapshot of one tree node (Listing 1 fields). capacity/used are bytes;
 * capacity 0 means "unbounded". */
typedef struct {
  int node_id;
  int storage_type;   /* NU_FILE / NU_HOST / NU_HBM / NU_SMEM */
  int physical_id;    /* device ordinal (HBM/SMEM), NUMA node or -1 */
  uint64_t capacity;  /* bytes, 0 = unbounded */
  uint64_t used;      /* bytes currently allocated by the library at this node */
  int processor_type; /* NU_PROC_* (leaf only) */
  int level;          /* 0 = root (slowest), increasing towards the leaves */
  int is_leaf;
  int parent;         /* -1 for the root */
  int num_children;
  int64_t block_bm, block_bn, block_bk; /* override from northup_tree_set_block, 0 = auto */
} northup_node_info;

/* ---------------------------------------------------------------- the tree */
/* Create an empty tree ("constructed by the runtime library at program
 * initialization").  *out receives the handle. */
int northup_tree_create(northup_tree_t* out);

/* Add a node under `parent` (-1 adds the root; only one root).  Listing 1,
 * P:76-92.  storage: NU_FILE/NU_HOST/NU_HBM/NU_SMEM.  physical_id: device
 * ordinal for NU_HBM/NU_SMEM (several HBM nodes may alias one ordinal:
 * "virtual siblings" for testing), else -1.  capacity_bytes: 0 = unbounded.
 * processor: NU_PROC_SM100 marks the leaf where computation happens (an HBM
 * node with a processor is a leaf whose kernel stages SMEM internally; an
 * SMEM node must be a child of an HBM node with the same physical_id).
 * *node_id receives the new node's id.  Levels are assigned as depth from
 * the root.  Fails with NU_ESTATE after finalize. */
int northup_tree_add_node(northup_tree_t t, int parent, int storage, int physical_id,
                          uint64_t capacity_bytes, int processor, int* node_id);

/* Manual block sizes for the chunks `node` hands to its children ("4k x 4k
 * in DRAM ... manually chosen"); 0 = let the planner decide. bm/bn/bk > 0 and, for
 * bk, a multiple of 4. */
int northup_tree_set_block(northup_tree_t t, int node, int64_t bm, int64_t bn, int64_t bk);

/* Adopt caller-owned device memory (e.g. a torch tensor) as the arena of an HBM
 * node instead of cudaMalloc. The arena must stay valid until destroy. */
int northup_tree_set_arena(northup_tree_t t, int node, void* dev_ptr, uint64_t bytes);

/* Register the caller-owned device buffer (M x N fp32, row-major) that
 * receives the whole C on this HBM node when northup_gemm_ex runs with
 * opts->replicate_result (S§8(e)).  HOST root, one process: the plan copies
 * every finished C piece from its sibling's HBM into every replica (peer
 * device-to-device copies over NVLink, issued as the piece drains, so they
 * overlap the rest of the GEMM).  Other trees: after the join (NCCL over
 * NVLink for distinct devices, device copies for siblings aliasing one
 * device).  NULL unregisters. */
int northup_tree_set_replica(northup_tree_t t, int node, void* dev_ptr, uint64_t bytes);

/* Validate the tree (P:95 level rule: every path from the root ends in a leaf
 * with a processor; storage levels only get faster towards the leaves), create
 * streams/events for every HBM node, and prepare the per-node arenas.
 * Needs the CUDA devices named by HBM nodes. */
int northup_tree_finalize(northup_tree_t t);

/* Free every library-owned buffer, stream, event and file. */
int northup_tree_destroy(northup_tree_t t);

/* ------------------------------------------ tree query API */
int northup_fetch_node_type(northup_tree_t t, int node, int* storage_type);
int northup_get_parent(northup_tree_t t, int node, int* parent);
/* Writes up to `cap` child ids into out[], the total count into *n. */
int northup_get_children_list(northup_tree_t t, int node, int* out, int cap, int* n);
int northup_get_level(northup_tree_t t, int node, int* level);
/* Number of levels below the root along the deepest path (root-only tree: 0). */
int northup_get_max_treelevel(northup_tree_t t, int* max_level);
int northup_get_num_nodes(northup_tree_t t, int* n);
int northup_get_node_info(northup_tree_t t, int node, northup_node_info* info);
/* Human-readable topology ("Northup can output the topology"); writes a
 * NUL-terminated string of at most n bytes; *n_needed (may be NULL) gets the
 * full length + 1. */
int northup_tree_print(northup_tree_t t, char* buf, size_t n, size_t* n_needed);
/* errno of the last failed file read / write / fdatasync of any FILE path in
 * this process (0 for an unexpected end of file); a failed call returns
 * NU_EIO and northup_last_error() names the operation.  Testing: the env var
 * NORTHUP_IO_FAULT="<read|write>:<eio|enospc|short|eof>:<n>" makes the n-th
 * pread (pwrite) of the process fail with EIO / ENOSPC, move half the bytes
 * (a short transfer, which the library completes) or return 0. */
int northup_last_io_errno(void);
/* What finalize measured about the tree's links (exec.cpp): *pcie_gbs = the
 * slowest local GPU's host->HBM rate with every local link busy in both
 * directions (64 MiB pinned copies; 0 = not measured: HBM root, no GPU worker,
 * or NORTHUP_CALIBRATE=0 — the planner then uses its nominal 49 GB/s);
 * *p2p_ok = 1 when every pair of distinct HBM devices has peer access (else
 * shared staging, S§8(f) NEXT-1, is not planned); *numa_bound = number of local
 * workers whose threads are bound to their GPU's NUMA node.  NU_ESTATE before
 * finalize. */
int northup_tree_link_info(northup_tree_t t, double* pcie_gbs, int* p2p_ok, int* numa_bound);

/* ---------------------------------------- unified data API (Table I) */
/* alloc(size, tree_node): pinned portable host memory at a NU_HOST node, a
 * created file at a NU_FILE node (`path_hint` directory via
 * northup_tree_set_file_dir), device memory at a NU_HBM node.  Counted in the
 * node's `used`; fails with NU_ENOMEM beyond its capacity. */
int northup_alloc(northup_tree_t t, uint64_t bytes, int node, northup_buf_t* out);
/* Directory for files created by northup_alloc at NU_FILE nodes (default /tmp). */
int northup_tree_set_file_dir(northup_tree_t t, const char* dir);
/* Wrap caller memory at a NU_HOST node (registered with cudaHostRegister if not
 * already pinned) — the caller keeps ownership. */
int northup_wrap_host(northup_tree_t t, int node, void* ptr, uint64_t bytes, northup_buf_t* out);
/* Wrap caller device memory at a NU_HBM node (the in-HBM reference, CS4). */
int northup_wrap_device(northup_tree_t t, int node, void* dev_ptr, uint64_t bytes,
                        northup_buf_t* out);
/* Open an existing file (or create it with `bytes` if absent) at a NU_FILE node.
 * Data is a dense row-major fp32 matrix at offset 0.  O_DIRECT is used when the
 * file system and alignment allow it, else buffered I/O. */
int northup_open_file(northup_tree_t t, int node, const char* path, uint64_t bytes,
                      northup_buf_t* out);
/* Properties of a handle: node, host/device pointer (NULL for files), size. */
int northup_buf_info(northup_buf_t b, int* node, void** ptr, uint64_t* bytes);
/* move_data(dst, src, size, offset, ...) (Table I, Listing 4):
 * copy `bytes` from src+src_off to dst+dst_off; the copy routine is picked from
 * the two nodes' storage types (file read/write, memcpy, cudaMemcpy). Synchronous. */
int northup_move_data(northup_tree_t t, northup_buf_t dst, uint64_t dst_off, northup_buf_t src,
                      uint64_t src_off, uint64_t bytes);
/* move_data_down (Table I): dst must live at the i-th child of src's node. */
int northup_move_data_down(northup_tree_t t, northup_buf_t dst, northup_buf_t src, uint64_t bytes,
                           uint64_t src_off, int child_index);
/* move_data_up (Table I): dst must live at the parent of src's node. */
int northup_move_data_up(northup_tree_t t, northup_buf_t dst, northup_buf_t src, uint64_t bytes,
                         uint64_t dst_off);
/* release(ptr) (Table I). Releasing a wrapped buffer unregisters only. */
int northup_release(northup_tree_t t, northup_buf_t b);

/* ------------------------------------------------------- the GEMM (§IV-A) */
typedef struct {
  int schedule;         /* NU_SCHED_AUTO / S1 / S2 / QUEUE / S2B */
  int replicate_result; /* 1: every HBM node's replica buffer (northup_tree_set_replica)
                           receives the whole C: pushed piece by piece during the call
                           (HOST root, one process) or gathered after the join */
  int64_t k_chunk;      /* K panel of one leaf launch and of one operand split (0 = 2048); the
                           TMEM accumulation inside a panel is 256 (R20) */
  int npass;            /* leaf split (R22): 0 = default (3); 3 = fp16 hi.hi + hi.lo +
                           lo.hi on the scaled split; 4 = + lo.lo; 1 = hi.hi only (negative test) */
  int resident;         /* 1: run the plan with operands already resident (in-HBM timing) */
  int collect_timing;   /* 1: record per-stage CUDA-event timings into the stats */
  int64_t a_panel_k;    /* FILE root only: A is stored K-panel-major (R15 preprocessing,
                           see northup_file_tile_kpanels) with this panel width; 0 = row-major */
  int graph;            /* 1: capture each GPU's op list into a CUDA graph and replay it when the
                           same GEMM (sizes, buffers, options) is called again — the recursion
                           unfolded into a dependency graph (P:230 future work); HOST/HBM roots */
  int shared_staging;   /* HOST root with G > 1 HBM siblings (S§8(f) NEXT-1): 0 = auto (on
                           when every sibling has a region of the same shape under S2), -1 = off.
                           Each sibling loads only 1/Pc of every A panel and 1/Pr of every B panel
                           over its PCIe link and pulls the rest from its grid-row / grid-column
                           peers' HBM (NVLink P2P; a local copy between virtual siblings).  C is
                           bitwise identical with and without it.  Disables `graph`. */
  int queue_tiles;      /* NU_SCHED_QUEUE: C tiles per HBM sibling (0 = 2); more tiles balance
                           better but stream more A/B bytes */
  int reserved[3];
} northup_gemm_opts;

typedef struct {
  double t_total_ms;     /* wall time of the call (host steady clock) */
  double t_plan_ms;      /* planner + partitioner (host) */
  double t_h2d_ms;       /* sum over GPUs of busy time of H2D copies (timing mode) */
  double t_compute_ms;   /* sum over GPUs of leaf-kernel busy time (timing mode) */
  double t_d2h_ms;       /* sum over GPUs of busy time of D2H copies (timing mode) */
  double t_io_ms;        /* file read/write time (host) */
  uint64_t bytes_h2d, bytes_d2h, bytes_d2d, bytes_file_read, bytes_file_write;
  int64_t leaf_launches; /* leaf kernels launched */
  int64_t copies;        /* copy operations issued */
  int64_t ops;           /* plan operations */
  int64_t bm, bn, bk;    /* blocks chosen at the HBM edge of GPU 0 */
  int64_t tail_k, strips;/* staggered-drain tail (S2) */
  int schedule;          /* schedule used */
  int num_gpus;          /* HBM siblings used */
  uint64_t hbm_peak_bytes; /* planned footprint at the HBM node of GPU 0 */
  int graph_replayed;    /* 1 when the call replayed CUDA graphs captured by an earlier call */
  int shared_staging;    /* 1 when the plan used NVLink-shared staging (opts->shared_staging) */
  uint64_t bytes_p2p;    /* bytes pulled from sibling HBM (shared staging), all GPUs */
  double t_p2p_ms;       /* sum over GPUs of busy time of sibling pulls (timing mode) */
  int64_t tasks;         /* NU_SCHED_QUEUE: C tiles */
  int64_t tasks_stolen;  /* NU_SCHED_QUEUE: tiles a sibling took from another sibling's queue */
  int file_direct_mode;  /* FILE root with HBM children (GDS edge): 1 = cuFile, 2 = pinned bounce */
  int bfirst_rows;       /* NU_SCHED_S2B: C rows computed while B streams (r1); 0 otherwise */
} northup_stats;

/* C = A.B (no alpha/beta; C overwritten — reading R3), A (M x K), B (K x N),
 * C (M x N), row-major and dense (ld = K, N, N), all resident at the ROOT node
 * (pinned host, file, or — for a single-node HBM tree — device memory).
 * Any M, N, K >= 0: M*N == 0 is a no-op; K == 0 sets C = 0. Synchronous: returns
 * when C is complete in the root tier. */
int northup_gemm(northup_tree_t t, northup_buf_t A, northup_buf_t B, northup_buf_t C, int64_t M,
                 int64_t N, int64_t K);
/* As northup_gemm with options (may be NULL) and statistics (may be NULL). */
int northup_gemm_ex(northup_tree_t t, northup_buf_t A, northup_buf_t B, northup_buf_t C, int64_t M,
                    int64_t N, int64_t K, const northup_gemm_opts* opts, northup_stats* stats);

/* ----------------------------------------------------- the leaf directly */
/* The SMEM/TMEM leaf on device pointers (CS4 in-HBM reference and tests):
 * C = A.B (accumulate = 0) or C += A.B (accumulate = 1), row-major, on `stream`
 * (a cudaStream_t, NULL = legacy default) of the CURRENT device ("C = AB").
 * Per K panel of k_chunk (0 = 2048) the operands are split into scaled fp16
 * hi/lo pairs (R22) in stream-ordered scratch the library owns
 * ((M + N) x panel x 4 bytes, freed on the stream), then multiplied with
 * tcgen05 MMAs.  A, B, C any alignment; N <= 49152; npass 0/3 = the product
 * split, 4 = + lo.lo, 1 = hi.hi only (negative test); other values NU_EINVAL.
 * Asynchronous: returns after the launches. */
int northup_leaf_gemm(const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
                      int64_t ldc, int64_t M, int64_t N, int64_t K, int accumulate, int64_t k_chunk,
                      int npass, void* stream);

/* --------------------------------------------------- plan introspection */
/* One operation of a plan.  op: NU_OP_COPY (2-D copy rows x cols floats from
 * src to dst), NU_OP_LEAF (C += / = A.B on the GPU), NU_OP_ZERO (C block = 0).
 * Buffers are plan-local ids (see northup_plan_buffer). */
#define NU_OP_COPY 0
#define NU_OP_LEAF 1
#define NU_OP_ZERO 2
#define NU_OP_IO_READ 3  /* file -> DRAM staging (pread), host I/O thread */
#define NU_OP_IO_WRITE 4 /* DRAM staging -> file (pwrite), host I/O thread */
#define NU_OP_SPLIT_B 6  /* split a resident B region in place into the leaf's fp16 hi/lo operand
                            (R22): dst_* = the region (rows = K rows of one panel,
                            cols = N), c_buf / c_off = its column exponents (ints); a LEAF op
                            whose src_buf >= 0 reads such a B, exponents at src_buf / src_off,
                            `rows` = exponents per K panel */
#define NU_OP_STENCIL 5  /* HotSpot-2D leaf (northup_hotspot): a_* = temperature in, b_* = power,
                            c_* = temperature out, all shaped like the m x n window; k = iterations;
                            src_off / dst_off = the window's grid row / column; rows x cols = grid */
typedef struct {
  int op;
  int worker;   /* GPU worker index (0 .. num_gpus-1) */
  int stream;   /* 0 = H2D, 1 = compute, 2 = D2H, 3 = file reads, 4 = D2D (sibling pulls), 5 = file writes */
  int accumulate;
  int src_buf, dst_buf; /* COPY */
  int a_buf, b_buf, c_buf; /* LEAF / ZERO(c) */
  int64_t src_off, dst_off, src_ld, dst_ld, rows, cols; /* COPY, element units */
  int64_t a_off, b_off, c_off, lda, ldb, ldc, m, n, k;  /* LEAF, element units */
  int ndeps;
  int deps[16]; /* indices of earlier ops this op must wait for (pruned per worker and stream;
                   may name another worker's op: shared-staging pulls) */
} northup_op;

typedef struct {
  int kind;       /* 0 = user A, 1 = user B, 2 = user C, 3 = node arena, 4 = DRAM staging,
                     5 = a sibling's replica of C (replicate_result pushes) */
  int node;       /* tree node the buffer lives at */
  int worker;     /* owning worker for arenas, -1 for user buffers */
  uint64_t bytes; /* size (arena: planned footprint) */
} northup_plan_buf;

typedef struct northup_plan_s* northup_plan_t;

/* Build (but do not run) the plan for an M x N x K GEMM on a finalized or
 * unfinalized tree.  Host-only; never touches a GPU. */
int northup_plan_create(northup_tree_t t, int64_t M, int64_t N, int64_t K,
                        const northup_gemm_opts* opts, northup_plan_t* out);
int northup_plan_num_ops(northup_plan_t p, int64_t* n);
int northup_plan_get_op(northup_plan_t p, int64_t i, northup_op* out);
int northup_plan_num_bufs(northup_plan_t p, int* n);
int northup_plan_get_buf(northup_plan_t p, int i, northup_plan_buf* out);
/* Same statistics the executor reports, predicted from the plan (bytes, blocks). */
int northup_plan_stats(northup_plan_t p, northup_stats* out);
int northup_plan_destroy(northup_plan_t p);

/* ------------------------------------------- file-root preprocessing (R15) */
/* P:353 "preprocessing the original file and reorganizing it ... for chunking":
 * rewrite a row-major M x K fp32 matrix file `src` as K-panel-major `dst`
 * (panel p = columns [p*panel_k, (p+1)*panel_k), row-major inside, panels
 * stored one after another; the last panel may be narrower), so that each
 * K panel of A is one sequential read.  Host-only; a one-time cost reported
 * separately from the GEMM (reading R15). */
int northup_file_tile_kpanels(const char* src, const char* dst, int64_t M, int64_t K,
                              int64_t panel_k);

/* -------------------------------------------------------- partitioner */
/* The 2-D grid Pr x Pc = G that minimises per-GPU H2D bytes 4K(M/Pr + N/Pc),
 * ties to more row splits; region r (row-major over the grid)
 * covers rows [*r0, *r1) and columns [*c0, *c1). */
int northup_partition(int G, int64_t M, int64_t N, int64_t K, int* Pr, int* Pc);
int northup_partition_region(int G, int64_t M, int64_t N, int64_t K, int r, int64_t* r0,
                             int64_t* r1, int64_t* c0, int64_t* c1);

/* ------------------------------------------ multi-process siblings (S§8(e)) */
/* One process per GPU (torchrun): every process builds the SAME tree (HOST
 * root -> G HBM children, node i on the GPU of process i) and calls
 * northup_tree_set_local(t, its HBM node) before finalize.  northup_gemm then
 * runs only that sibling's share of the plan, and A, B, C passed to it hold
 * only this sibling's strips: A rows [r0, r1) (ld K), B columns [c0, c1)
 * (ld c1 - c0), C the (r1 - r0) x (c1 - c0) region (ld c1 - c0), with the region
 * from northup_partition_region(G, M, N, K, index of the node among the root's
 * children).  Without shared staging no peer is involved.  With shared staging
 * (NEXT-1, opts->shared_staging) the pulls read the peers' HBM: before the
 * first GEMM of a shape every process calls northup_peer_export (plans the GEMM,
 * allocates its arena and flag words, writes a blob of CUDA IPC handles into
 * `blob`, `cap` >= *len bytes; *len is set even when cap is too small), the
 * blobs are exchanged between processes by the caller (e.g. all_gather_object)
 * and each process imports every other sibling's blob with northup_peer_import
 * (worker = that sibling's index).  Export/import are collective: every
 * process does them for the same GEMM, after its previous GEMM returned.
 * Cross-sibling dependencies are device-side waits on flag words (no host
 * blocking); each call ends with a device-side join of all siblings.
 * Errors: NU_ESTATE when called out of order or when northup_gemm runs a
 * shared plan without a matching export/import; NU_ECUDA for IPC failures
 * (e.g. a blob from this same process). */
int northup_tree_set_local(northup_tree_t t, int node);
int northup_peer_export(northup_tree_t t, int64_t M, int64_t N, int64_t K,
                        const northup_gemm_opts* opts, void* blob, uint64_t cap, uint64_t* len);
int northup_peer_import(northup_tree_t t, int worker, const void* blob, uint64_t len);

/* ------------------------------------------ HotSpot-2D stencil (S§8(f) NEXT-3) */
/* The paper's second case study (§IV-B): HotSpot-2D [18] thermal
 * simulation over the same tree.  One iteration updates every cell (r, c) of
 * the rows x cols fp32 temperature grid T with power grid P:
 *   T'[r,c] = T + cap_1 * (P + (T[r+1,c] + T[r-1,c] - 2T) * ry_1
 *                            + (T[r,c+1] + T[r,c-1] - 2T) * rx_1 + (amb - T) * rz_1)
 * with out-of-grid neighbours replaced by the cell itself (RH1), in
 * fp32 through one fixed sequence of the expanded form (RH4):
 *   kt = 1 - cap_1 (2 rx_1 + 2 ry_1 + rz_1), kx = cap_1 rx_1, ky = cap_1 ry_1,
 *   kq = cap_1 rz_1 amb (each rounded once to fp32), q = fma(cap_1, P, kq),
 *   T' = fma(ky, S + N, fma(kx, E + W, fma(kt, T, q)))
 * (round-to-nearest; identical on every path, so in-HBM and out-of-core runs
 * agree bit for bit; within RH3's bound of the fp64 definition). */
typedef struct {
  float cap_1, rx_1, ry_1, rz_1, amb;
} northup_hotspot_coeffs;

/* [18]'s chip model with the cell pitch fixed at its 1024-cell value (reading
 * RH2, so the explicit scheme is stable at any grid size), rounded to fp32. */
int northup_hotspot_default_coeffs(int64_t rows, int64_t cols, northup_hotspot_coeffs* out);

typedef struct {
  int64_t block;      /* HBM-level block edge in cells ("8k x 8k blocking"), 0 = planner */
  int64_t halo;       /* iterations per visit of a block to HBM = its border width, 0 = planner */
  int leaf_iters;     /* iterations per leaf launch (1..8), 0 = 8 */
  int collect_timing; /* 1: per-stream busy times into the stats */
  int reserved[4];
} northup_hotspot_opts;

/* The leaf on device pointers: `iters` (1..8) iterations on the wm x wn window
 * whose top-left cell is (gy0, gx0) of a rows x cols grid.  tin/pw/tout are
 * window-shaped (leading dimensions ldt/ldp/ldo >= wn).  Writes only the valid
 * region of tout: the window shrunk by `iters` cells on each side that is not
 * a grid edge.  Asynchronous on `stream` (current device).  NU_EINVAL for a
 * window outside the grid or iters outside 1..8. */
int northup_hotspot_leaf(const float* tin, int64_t ldt, const float* pw, int64_t ldp, float* tout,
                         int64_t ldo, int64_t wm, int64_t wn, int64_t gy0, int64_t gx0,
                         int64_t rows, int64_t cols, int iters, const northup_hotspot_coeffs* k,
                         void* stream);

/* `iters` iterations of HotSpot-2D on the tree: T (input, unchanged), P and
 * Tout, each rows x cols fp32 row-major, live at the ROOT (pinned host, or
 * device memory for a single-node HBM tree).  Synchronous.  A HOST root splits
 * the grid into blocks that move down to the HBM siblings with a border of
 * `halo` cells (the four borders of P:317, strided rows copied by the DMA
 * engine), iterate `halo` times there and move back up; passes alternate
 * between Tout and a library-owned pinned scratch grid.  k NULL = defaults.
 * iters == 0 copies T to Tout. */
int northup_hotspot(northup_tree_t t, northup_buf_t T, northup_buf_t P, northup_buf_t Tout,
                    int64_t rows, int64_t cols, int64_t iters, const northup_hotspot_coeffs* k,
                    const northup_hotspot_opts* opts, northup_stats* stats);
/* Build (not run) the HotSpot-2D plan; introspect it with northup_plan_*. */
int northup_hotspot_plan(northup_tree_t t, int64_t rows, int64_t cols, int64_t iters,
                         const northup_hotspot_opts* opts, northup_plan_t* out);

/* ------------------------------------------------------------ misc */
const char* northup_last_error(void);
int northup_version(void);
/* Number of CUDA devices visible (0 without a GPU; never fails). */
int northup_device_count(void);

#ifdef __cplusplus
}
#endif
#endif /* NORTHUP_H */
