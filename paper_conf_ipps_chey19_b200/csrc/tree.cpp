// Tree descriptor (Listing 1), tree query API, topology
// printout and the unified data-management API (Table I, P:264-272;
// Listing 4).
#include <errno.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <atomic>
#include <fcntl.h>
#include <stdarg.h>
#include <stdio.h>
#include <string.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <string>

#include "northup_internal.h"

namespace nu {
static std::atomic<int> g_io_errno{0};
static std::atomic<long long> g_io_calls[2];

void note_io_errno(int e) { g_io_errno.store(e); }

ssize_t pio(int fd, void* p, size_t n, uint64_t off, bool write) {
  static const char* spec = getenv("NORTHUP_IO_FAULT");
  if (spec && *spec) {
    char op[16] = {}, kind[16] = {};
    long long nth = 0;
    if (sscanf(spec, "%15[^:]:%15[^:]:%lld", op, kind, &nth) == 3 && (strcmp(op, "write") == 0) == write) {
      const long long k = g_io_calls[write ? 1 : 0].fetch_add(1) + 1;
      if (k == nth) {
        if (strcmp(kind, "eio") == 0) {
          errno = EIO;
          return -1;
        }
        if (strcmp(kind, "enospc") == 0) {
          errno = ENOSPC;
          return -1;
        }
        if (strcmp(kind, "eof") == 0) return 0;
        if (strcmp(kind, "short") == 0 && n > 1) n /= 2;
      }
    }
  }
  return write ? pwrite(fd, p, n, static_cast<off_t>(off)) : pread(fd, p, n, static_cast<off_t>(off));
}
}  // namespace nu


extern "C" int northup_last_io_errno(void);

namespace nu {

static thread_local char g_err[1024] = "";

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

int fail(int code, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
  return code;
}

int cuda_fail(cudaError_t e, const char* what) {
  return fail(NU_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

static bool valid_node(const northup_tree_s* t, int node) {
  return t && node >= 0 && node < static_cast<int>(t->nodes.size());
}

// Level rule: level 0 = slowest storage (the root), larger = faster.
// Storage "speed rank" used to check that every edge goes to faster memory.
static int speed_rank(int storage) {
  switch (storage) {
    case NU_FILE: return 0;
    case NU_HOST: return 1;
    case NU_HBM: return 2;
    case NU_SMEM: return 3;
  }
  return -1;
}

int validate_tree(const northup_tree_s* t) {
  if (!t || t->nodes.empty()) return fail(NU_EINVAL, "tree has no nodes");
  for (const Node& n : t->nodes) {
    const bool leaf = n.children.empty();
    if (leaf && n.processor == NU_PROC_NONE)
      return fail(NU_EINVAL, "leaf node %d has no processor (P:95: computation happens at leafs)",
                  n.id);
    if (!leaf && n.processor != NU_PROC_NONE)
      return fail(NU_ENOTSUP, "processor at inner node %d is not supported (no CPU leaf on the path)",
                  n.id);
    if (n.processor == NU_PROC_SM100 && n.storage != NU_HBM && n.storage != NU_SMEM)
      return fail(NU_EINVAL, "SM100 processor attached to node %d that is not HBM/SMEM", n.id);
    if (n.storage == NU_SMEM) {
      if (!leaf) return fail(NU_EINVAL, "SMEM node %d must be a leaf", n.id);
      if (n.parent < 0 || t->nodes[n.parent].storage != NU_HBM ||
          t->nodes[n.parent].phys != n.phys)
        return fail(NU_EINVAL, "SMEM leaf %d must hang under the HBM node of the same GPU", n.id);
    }
    if ((n.storage == NU_HBM || n.storage == NU_SMEM) && n.phys < 0)
      return fail(NU_EINVAL, "HBM/SMEM node %d needs a device ordinal as physical_id", n.id);
    for (int c : n.children) {
      if (speed_rank(t->nodes[c].storage) <= speed_rank(n.storage) &&
          !(n.storage == NU_HOST && t->nodes[c].storage == NU_HOST))
        return fail(NU_EINVAL, "edge %d -> %d does not go to faster memory (P:95)", n.id, c);
    }
  }
  return 0;
}

}  // namespace nu

using namespace nu;

extern "C" {

const char* northup_last_error(void) { return nu::g_err; }
int northup_version(void) { return NORTHUP_VERSION; }

int northup_device_count(void) {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

int northup_tree_create(northup_tree_t* out) {
  if (!out) return fail(NU_EINVAL, "out is NULL");
  *out = new northup_tree_s();
  return 0;
}

int northup_tree_add_node(northup_tree_t t, int parent, int storage, int physical_id,
                          uint64_t capacity_bytes, int processor, int* node_id) {
  if (!t) return fail(NU_EINVAL, "tree is NULL");
  if (t->finalized) return fail(NU_ESTATE, "tree already finalized");
  if (storage < NU_FILE || storage > NU_SMEM) return fail(NU_EINVAL, "unknown storage type %d", storage);
  if (processor != NU_PROC_NONE && processor != NU_PROC_SM100)
    return fail(NU_EINVAL, "unknown processor type %d", processor);
  if (parent == -1) {
    if (!t->nodes.empty()) return fail(NU_EINVAL, "the tree already has a root");
  } else if (!valid_node(t, parent)) {
    return fail(NU_EINVAL, "unknown parent node %d", parent);
  }
  Node n;
  n.id = static_cast<int>(t->nodes.size());
  n.storage = storage;
  n.phys = physical_id;
  n.capacity = capacity_bytes;
  n.processor = processor;
  n.parent = parent;
  n.level = parent < 0 ? 0 : t->nodes[parent].level + 1;
  t->nodes.push_back(n);
  if (parent >= 0) t->nodes[parent].children.push_back(n.id);
  if (node_id) *node_id = n.id;
  return 0;
}

int northup_tree_set_block(northup_tree_t t, int node, int64_t bm, int64_t bn, int64_t bk) {
  if (!valid_node(t, node)) return fail(NU_EINVAL, "unknown node %d", node);
  if (bm < 0 || bn < 0 || bk < 0) return fail(NU_EINVAL, "negative block size");
  if (bk % 4) return fail(NU_EINVAL, "bk must be a multiple of 4 (16-byte TMA rows)");
  Node& n = t->nodes[node];
  n.bm = bm;
  n.bn = bn;
  n.bk = bk;
  return 0;
}

int northup_tree_set_arena(northup_tree_t t, int node, void* dev_ptr, uint64_t bytes) {
  if (!valid_node(t, node)) return fail(NU_EINVAL, "unknown node %d", node);
  Node& n = t->nodes[node];
  if (n.storage != NU_HBM) return fail(NU_EINVAL, "arena only for HBM nodes");
  if (!dev_ptr || bytes == 0) return fail(NU_EINVAL, "empty arena");
  if (reinterpret_cast<uintptr_t>(dev_ptr) % 256) return fail(NU_EINVAL, "arena must be 256-B aligned");
  if (n.capacity && bytes > n.capacity) return fail(NU_ENOMEM, "arena larger than node capacity");
  if (n.arena_owned && n.arena) {
    cudaSetDevice(n.phys);
    cudaFree(n.arena);
  }
  n.arena = dev_ptr;
  n.arena_bytes = bytes;
  n.arena_owned = false;
  return 0;
}

int northup_tree_set_local(northup_tree_t t, int node) {
  if (!t) return fail(NU_EINVAL, "tree is NULL");
  if (t->finalized) return fail(NU_ESTATE, "set_local must precede finalize");
  if (!valid_node(t, node) || t->nodes[node].storage != NU_HBM)
    return fail(NU_EINVAL, "node %d is not an HBM node", node);
  const int root = 0;
  if (t->nodes[root].storage != NU_HOST || t->nodes[node].parent != root)
    return fail(NU_ENOTSUP, "multi-process siblings need a HOST root with HBM children");
  t->local_node = node;
  return 0;
}

int northup_tree_finalize(northup_tree_t t) {
  if (!t) return fail(NU_EINVAL, "tree is NULL");
  if (t->finalized) return fail(NU_ESTATE, "tree already finalized");
  int rc = validate_tree(t);
  if (rc) return rc;
  rc = finalize_workers(t);
  if (rc) return rc;
  t->finalized = true;
  return 0;
}

int northup_release(northup_tree_t t, northup_buf_t b);

int northup_tree_destroy(northup_tree_t t) {
  if (!t) return fail(NU_EINVAL, "tree is NULL");
  while (!t->bufs.empty()) northup_release(t, t->bufs.back());
  destroy_nccl(t);
  destroy_graphs(t);
  destroy_peers(t);
  destroy_workers(t);
  for (Node& n : t->nodes) {
    if (n.arena_owned && n.arena) {
      if (n.storage == NU_HOST) {
        cudaFreeHost(n.arena);
      } else {
        cudaSetDevice(n.phys);
        cudaFree(n.arena);
      }
    }
    n.arena = nullptr;
  }
  delete t;
  return 0;
}

// ------------------------------------------------------------- queries
int northup_fetch_node_type(northup_tree_t t, int node, int* storage_type) {
  if (!valid_node(t, node) || !storage_type) return fail(NU_EINVAL, "bad node or NULL out");
  *storage_type = t->nodes[node].storage;
  return 0;
}

int northup_get_parent(northup_tree_t t, int node, int* parent) {
  if (!valid_node(t, node) || !parent) return fail(NU_EINVAL, "bad node or NULL out");
  *parent = t->nodes[node].parent;
  return 0;
}

int northup_get_children_list(northup_tree_t t, int node, int* out, int cap, int* n) {
  if (!valid_node(t, node) || !n) return fail(NU_EINVAL, "bad node or NULL out");
  const auto& ch = t->nodes[node].children;
  *n = static_cast<int>(ch.size());
  for (int i = 0; i < cap && i < *n; ++i) {
    if (!out) return fail(NU_EINVAL, "NULL list with cap > 0");
    out[i] = ch[i];
  }
  return 0;
}

int northup_get_level(northup_tree_t t, int node, int* level) {
  if (!valid_node(t, node) || !level) return fail(NU_EINVAL, "bad node or NULL out");
  *level = t->nodes[node].level;
  return 0;
}

int northup_get_max_treelevel(northup_tree_t t, int* max_level) {
  if (!t || !max_level) return fail(NU_EINVAL, "NULL argument");
  if (t->nodes.empty()) return fail(NU_EINVAL, "empty tree");
  int m = 0;
  for (const Node& n : t->nodes) m = std::max(m, n.level);
  *max_level = m;
  return 0;
}

int northup_get_num_nodes(northup_tree_t t, int* n) {
  if (!t || !n) return fail(NU_EINVAL, "NULL argument");
  *n = static_cast<int>(t->nodes.size());
  return 0;
}

int northup_get_node_info(northup_tree_t t, int node, northup_node_info* info) {
  if (!valid_node(t, node) || !info) return fail(NU_EINVAL, "bad node or NULL out");
  const Node& n = t->nodes[node];
  info->node_id = n.id;
  info->storage_type = n.storage;
  info->physical_id = n.phys;
  info->capacity = n.capacity;
  info->used = n.used;
  info->processor_type = n.processor;
  info->level = n.level;
  info->is_leaf = n.children.empty() ? 1 : 0;
  info->parent = n.parent;
  info->num_children = static_cast<int>(n.children.size());
  info->block_bm = n.bm;
  info->block_bn = n.bn;
  info->block_bk = n.bk;
  return 0;
}

static const char* storage_name(int s) {
  switch (s) {
    case NU_FILE: return "FILE";
    case NU_HOST: return "HOST";
    case NU_HBM: return "HBM";
    case NU_SMEM: return "SMEM";
  }
  return "?";
}

static void fmt_bytes(char* b, size_t n, uint64_t v) {
  if (v == 0) snprintf(b, n, "unbounded");
  else if (v % (1ull << 30) == 0) snprintf(b, n, "%llu GiB", (unsigned long long)(v >> 30));
  else if (v % (1ull << 20) == 0) snprintf(b, n, "%llu MiB", (unsigned long long)(v >> 20));
  else snprintf(b, n, "%llu B", (unsigned long long)v);
}

static void print_node(const northup_tree_s* t, int id, int depth, std::string& out) {
  const Node& n = t->nodes[id];
  char cap[64], line[256];
  fmt_bytes(cap, sizeof cap, n.capacity);
  snprintf(line, sizeof line, "%*s[%d] level %d %s phys=%d cap=%s used=%llu%s%s\n", depth * 2, "",
           n.id, n.level, storage_name(n.storage), n.phys, cap, (unsigned long long)n.used,
           n.processor == NU_PROC_SM100 ? " proc=SM100" : "", n.children.empty() ? " (leaf)" : "");
  out += line;
  for (int c : n.children) print_node(t, c, depth + 1, out);
}

int northup_tree_link_info(northup_tree_t t, double* pcie_gbs, int* p2p_ok, int* numa_bound) {
  using namespace nu;
  if (!t) return fail(NU_EINVAL, "null tree");
  if (!t->finalized) return fail(NU_ESTATE, "tree not finalized");
  if (pcie_gbs) *pcie_gbs = t->pcie_gbs;
  if (p2p_ok) *p2p_ok = t->p2p_ok ? 1 : 0;
  if (numa_bound) {
    int n = 0;
    for (const auto& c : t->worker_cpus) n += c.empty() ? 0 : 1;
    *numa_bound = n;
  }
  return 0;
}

int northup_tree_print(northup_tree_t t, char* buf, size_t n, size_t* n_needed) {
  if (!t) return fail(NU_EINVAL, "tree is NULL");
  std::string s;
  if (!t->nodes.empty()) print_node(t, 0, 0, s);
  if (n_needed) *n_needed = s.size() + 1;
  if (buf && n) {
    size_t k = std::min(n - 1, s.size());
    memcpy(buf, s.data(), k);
    buf[k] = 0;
  }
  return 0;
}

// ------------------------------------------------- unified data API (Table I)
static int new_buf(northup_tree_t t, int node, northup_buf_t* out, northup_buf_s** b) {
  if (!valid_node(t, node)) return fail(NU_EINVAL, "unknown node %d", node);
  if (!out) return fail(NU_EINVAL, "out is NULL");
  *b = new northup_buf_s();
  (*b)->tree = t;
  (*b)->node = node;
  (*b)->storage = t->nodes[node].storage;
  return 0;
}

static int capacity_check(northup_tree_t t, int node, uint64_t bytes) {
  const Node& n = t->nodes[node];
  if (n.capacity && n.used + bytes > n.capacity)
    return fail(NU_ENOMEM, "node %d: %llu B requested, %llu of %llu B in use", node,
                (unsigned long long)bytes, (unsigned long long)n.used,
                (unsigned long long)n.capacity);
  return 0;
}

int northup_tree_set_file_dir(northup_tree_t t, const char* dir) {
  if (!t || !dir || !*dir) return fail(NU_EINVAL, "bad directory");
  t->file_dir = dir;
  return 0;
}

// alloc(size, tree_node) (Table I; "allocates space on a disk
// drive by generating a file ... return a void pointer" to the fd).
int northup_alloc(northup_tree_t t, uint64_t bytes, int node, northup_buf_t* out) {
  northup_buf_s* b = nullptr;
  int rc = new_buf(t, node, out, &b);
  if (rc) return rc;
  if ((rc = capacity_check(t, node, bytes))) {
    delete b;
    return rc;
  }
  Node& n = t->nodes[node];
  b->bytes = bytes;
  b->owned = true;
  if (n.storage == NU_HOST) {
    cudaError_t e = cudaHostAlloc(&b->ptr, bytes ? bytes : 1, cudaHostAllocPortable);
    if (e != cudaSuccess) {
      delete b;
      return fail(NU_ENOMEM, "cudaHostAlloc(%llu): %s", (unsigned long long)bytes,
                  cudaGetErrorString(e));
    }
  } else if (n.storage == NU_HBM) {
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(n.phys);
    cudaError_t e = cudaMalloc(&b->ptr, bytes ? bytes : 1);
    cudaSetDevice(prev);
    if (e != cudaSuccess) {
      delete b;
      return fail(NU_ENOMEM, "cudaMalloc(%llu) on device %d: %s", (unsigned long long)bytes, n.phys,
                  cudaGetErrorString(e));
    }
  } else if (n.storage == NU_FILE) {
    // D4 file registry: the tree remembers created files for cleanup.
    static int counter = 0;
    char path[4096];
    snprintf(path, sizeof path, "%s/northup_%d_%p_%d.bin", t->file_dir.c_str(), (int)getpid(),
             (void*)t, __atomic_fetch_add(&counter, 1, __ATOMIC_RELAXED));
    int fd = open(path, O_RDWR | O_CREAT | O_TRUNC, 0600);
    if (fd < 0) {
      delete b;
      return fail(NU_EIO, "open(%s): %s", path, strerror(errno));
    }
    if (ftruncate(fd, static_cast<off_t>(bytes)) != 0) {
      int err = errno;
      close(fd);
      unlink(path);
      delete b;
      return fail(NU_EIO, "ftruncate(%s): %s", path, strerror(err));
    }
    b->fd = fd;
    b->direct_fd = open(path, O_RDWR | O_DIRECT);
    b->path = path;
  } else {
    delete b;
    return fail(NU_EINVAL, "cannot allocate at an SMEM node (managed by the leaf kernel)");
  }
  n.used += bytes;
  t->bufs.push_back(b);
  *out = b;
  return 0;
}

int northup_wrap_host(northup_tree_t t, int node, void* ptr, uint64_t bytes, northup_buf_t* out) {
  northup_buf_s* b = nullptr;
  int rc = new_buf(t, node, out, &b);
  if (rc) return rc;
  if (t->nodes[node].storage != NU_HOST) {
    delete b;
    return fail(NU_EINVAL, "wrap_host needs a HOST node");
  }
  if (!ptr && bytes) {
    delete b;
    return fail(NU_EINVAL, "NULL pointer");
  }
  b->ptr = ptr;
  b->bytes = bytes;
  if (ptr && bytes) {
    cudaPointerAttributes attr;
    cudaError_t e = cudaPointerGetAttributes(&attr, ptr);
    const bool pinned = e == cudaSuccess && attr.type == cudaMemoryTypeHost;
    cudaGetLastError();
    if (!pinned) {
      e = cudaHostRegister(ptr, bytes, cudaHostRegisterPortable);
      if (e != cudaSuccess) {
        cudaGetLastError();
        delete b;
        return fail(NU_ECUDA, "cudaHostRegister(%llu B): %s", (unsigned long long)bytes,
                    cudaGetErrorString(e));
      }
      b->registered = true;
    }
  }
  t->bufs.push_back(b);
  *out = b;
  return 0;
}

int northup_wrap_device(northup_tree_t t, int node, void* dev_ptr, uint64_t bytes,
                        northup_buf_t* out) {
  northup_buf_s* b = nullptr;
  int rc = new_buf(t, node, out, &b);
  if (rc) return rc;
  if (t->nodes[node].storage != NU_HBM) {
    delete b;
    return fail(NU_EINVAL, "wrap_device needs an HBM node");
  }
  if (!dev_ptr && bytes) {
    delete b;
    return fail(NU_EINVAL, "NULL pointer");
  }
  b->ptr = dev_ptr;
  b->bytes = bytes;
  t->bufs.push_back(b);
  *out = b;
  return 0;
}

int northup_open_file(northup_tree_t t, int node, const char* path, uint64_t bytes,
                      northup_buf_t* out) {
  northup_buf_s* b = nullptr;
  int rc = new_buf(t, node, out, &b);
  if (rc) return rc;
  if (t->nodes[node].storage != NU_FILE || !path) {
    delete b;
    return fail(NU_EINVAL, "open_file needs a FILE node and a path");
  }
  int fd = open(path, O_RDWR | O_CREAT, 0600);
  if (fd < 0) {
    delete b;
    return fail(NU_EIO, "open(%s): %s", path, strerror(errno));
  }
  struct stat st;
  if (fstat(fd, &st) == 0 && static_cast<uint64_t>(st.st_size) < bytes) {
    if (ftruncate(fd, static_cast<off_t>(bytes)) != 0) {
      int err = errno;
      close(fd);
      delete b;
      return fail(NU_EIO, "ftruncate(%s): %s", path, strerror(err));
    }
  }
  b->fd = fd;
  b->direct_fd = open(path, O_RDWR | O_DIRECT);   // -1 where O_DIRECT is unsupported (tmpfs)
  b->bytes = bytes;
  b->path = path;
  t->bufs.push_back(b);
  *out = b;
  return 0;
}

int northup_buf_info(northup_buf_t b, int* node, void** ptr, uint64_t* bytes) {
  if (!b) return fail(NU_EINVAL, "buffer is NULL");
  if (node) *node = b->node;
  if (ptr) *ptr = b->ptr;
  if (bytes) *bytes = b->bytes;
  return 0;
}


// Listing 4: file_write = lseek + write; we use pread/pwrite
// loops (positional, restartable on short transfers).
static int file_rw(int fd, void* buf, uint64_t count, uint64_t offset, bool write) {
  uint8_t* p = static_cast<uint8_t*>(buf);
  while (count) {
    ssize_t r = nu::pio(fd, p, count, offset, write);
    if (r < 0) {
      if (errno == EINTR) continue;
      const int err = errno;
      nu::note_io_errno(err);
      return fail(NU_EIO, "%s: %s", write ? "pwrite" : "pread", strerror(err));
    }
    if (r == 0) {
      nu::note_io_errno(0);
      return fail(NU_EIO, "%s: unexpected end of file", write ? "pwrite" : "pread");
    }
    p += r;
    count -= static_cast<uint64_t>(r);
    offset += static_cast<uint64_t>(r);
  }
  return 0;
}

// move_data (Table I; Listing 4): inspect the source and
// destination node types and pick the copy routine.
int northup_move_data(northup_tree_t t, northup_buf_t dst, uint64_t dst_off, northup_buf_t src,
                      uint64_t src_off, uint64_t bytes) {
  if (!t || !dst || !src) return fail(NU_EINVAL, "NULL argument");
  if (dst->tree != t || src->tree != t) return fail(NU_EINVAL, "buffer from another tree");
  if (dst_off + bytes > dst->bytes || src_off + bytes > src->bytes)
    return fail(NU_EINVAL, "range exceeds buffer");
  if (bytes == 0) return 0;
  const int ds = dst->storage, ss = src->storage;
  if (ds == NU_FILE && ss == NU_FILE) {
    // file -> file through a bounce buffer
    std::vector<uint8_t> tmp(std::min<uint64_t>(bytes, 64ull << 20));
    uint64_t done = 0;
    while (done < bytes) {
      uint64_t k = std::min<uint64_t>(tmp.size(), bytes - done);
      int rc = file_rw(src->fd, tmp.data(), k, src_off + done, false);
      if (!rc) rc = file_rw(dst->fd, tmp.data(), k, dst_off + done, true);
      if (rc) return rc;
      done += k;
    }
    return 0;
  }
  if (ds == NU_FILE) {   // memory -> file  (Listing 4: file_write)
    if (ss == NU_HOST) return file_rw(dst->fd, static_cast<uint8_t*>(src->ptr) + src_off, bytes, dst_off, true);
    std::vector<uint8_t> tmp(bytes);
    cudaError_t e = cudaMemcpy(tmp.data(), static_cast<uint8_t*>(src->ptr) + src_off, bytes,
                               cudaMemcpyDefault);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy D2H");
    return file_rw(dst->fd, tmp.data(), bytes, dst_off, true);
  }
  if (ss == NU_FILE) {   // file -> memory
    if (ds == NU_HOST) return file_rw(src->fd, static_cast<uint8_t*>(dst->ptr) + dst_off, bytes, src_off, false);
    std::vector<uint8_t> tmp(bytes);
    int rc = file_rw(src->fd, tmp.data(), bytes, src_off, false);
    if (rc) return rc;
    cudaError_t e = cudaMemcpy(static_cast<uint8_t*>(dst->ptr) + dst_off, tmp.data(), bytes,
                               cudaMemcpyDefault);
    return e == cudaSuccess ? 0 : cuda_fail(e, "cudaMemcpy H2D");
  }
  if (ds == NU_HOST && ss == NU_HOST) {
    memmove(static_cast<uint8_t*>(dst->ptr) + dst_off, static_cast<uint8_t*>(src->ptr) + src_off,
            bytes);
    return 0;
  }
  // HOST <-> HBM, HBM <-> HBM: the CUDA copy engines (UVA picks the direction).
  cudaError_t e = cudaMemcpy(static_cast<uint8_t*>(dst->ptr) + dst_off,
                             static_cast<uint8_t*>(src->ptr) + src_off, bytes, cudaMemcpyDefault);
  return e == cudaSuccess ? 0 : cuda_fail(e, "cudaMemcpy");
}

int northup_move_data_down(northup_tree_t t, northup_buf_t dst, northup_buf_t src, uint64_t bytes,
                           uint64_t src_off, int child_index) {
  if (!t || !dst || !src) return fail(NU_EINVAL, "NULL argument");
  const auto& ch = t->nodes[src->node].children;
  if (child_index < 0 || child_index >= static_cast<int>(ch.size()) || ch[child_index] != dst->node)
    return fail(NU_EINVAL, "dst does not live at child %d of node %d", child_index, src->node);
  return northup_move_data(t, dst, 0, src, src_off, bytes);
}

int northup_move_data_up(northup_tree_t t, northup_buf_t dst, northup_buf_t src, uint64_t bytes,
                         uint64_t dst_off) {
  if (!t || !dst || !src) return fail(NU_EINVAL, "NULL argument");
  if (t->nodes[src->node].parent != dst->node)
    return fail(NU_EINVAL, "dst does not live at the parent of node %d", src->node);
  return northup_move_data(t, dst, dst_off, src, 0, bytes);
}

int northup_release(northup_tree_t t, northup_buf_t b) {
  if (!t || !b) return fail(NU_EINVAL, "NULL argument");
  auto it = std::find(t->bufs.begin(), t->bufs.end(), b);
  if (it == t->bufs.end()) return fail(NU_EINVAL, "buffer does not belong to this tree");
  t->bufs.erase(it);
  Node& n = t->nodes[b->node];
  if (b->owned) {
    if (b->storage == NU_HOST && b->ptr) cudaFreeHost(b->ptr);
    if (b->storage == NU_HBM && b->ptr) {
      int prev = 0;
      cudaGetDevice(&prev);
      cudaSetDevice(n.phys);
      cudaFree(b->ptr);
      cudaSetDevice(prev);
    }
    if (b->storage == NU_FILE) {
      if (b->fd >= 0) close(b->fd);
      if (b->direct_fd >= 0) close(b->direct_fd);
      if (!b->path.empty()) unlink(b->path.c_str());
      b->fd = -1;
    }
    n.used = n.used >= b->bytes ? n.used - b->bytes : 0;
  } else {
    if (b->registered && b->ptr) cudaHostUnregister(b->ptr);
    if (b->storage == NU_FILE && b->fd >= 0) close(b->fd);
    if (b->storage == NU_FILE && b->direct_fd >= 0) close(b->direct_fd);
  }
  delete b;
  return 0;
}

}  // extern "C"

extern "C" int northup_last_io_errno(void) { return nu::g_io_errno.load(); }
