// Plan builder shared by the GEMM planner (plan.cpp) and the HotSpot-2D
// planner (hotspot_plan.cpp): ops are appended in plan order and each op's
// dependencies are derived from the exact 2-D regions it reads and writes.
#pragma once

#include <algorithm>
#include <initializer_list>
#include <utility>
#include <vector>

#include "northup_internal.h"

namespace nu {

inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline int64_t rup(int64_t a, int64_t b) { return cdiv(a, b) * b; }
inline int64_t pad_ld(int64_t n) { return std::max<int64_t>(32, rup(n, 32)); }  // 128-B rows

struct Access {
  int op;
  int stream;
  int64_t lo, hi;      // bounding element interval
  int64_t off, ld, rows, cols;
  bool write;
};

// Do two 2-D regions of one buffer overlap?  Exact rectangle test when both
// use the same leading dimension and stay inside it, else the bounding
// intervals (conservative).
inline bool overlaps(const Access& p, int64_t lo, int64_t hi, int64_t off, int64_t ld, int64_t rows,
                     int64_t cols) {
  if (p.hi <= lo || hi <= p.lo) return false;
  if (p.ld != ld || ld <= 0) return true;
  const int64_t pr = p.off / ld, pc = p.off % ld, r = off / ld, c = off % ld;
  if (pc + p.cols > ld || c + cols > ld) return true;
  return pr < r + rows && r < pr + p.rows && pc < c + cols && c < pc + p.cols;
}

inline northup_op make_copy(int worker, int stream, int src, int64_t src_off, int64_t src_ld, int dst,
                     int64_t dst_off, int64_t dst_ld, int64_t rows, int64_t cols) {
  northup_op o{};
  o.op = NU_OP_COPY;
  o.worker = worker;
  o.stream = stream;
  o.src_buf = src;
  o.dst_buf = dst;
  o.src_off = src_off;
  o.dst_off = dst_off;
  o.src_ld = src_ld;
  o.dst_ld = dst_ld;
  o.rows = rows;
  o.cols = cols;
  o.a_buf = o.b_buf = o.c_buf = -1;
  return o;
}

struct Builder {
  Plan* P;
  // GEMM: root-tier regions of different siblings are disjoint by construction,
  // so user-buffer accesses never order two siblings.  HotSpot halos overlap
  // across siblings: false there.
  bool user_disjoint = true;
  std::vector<std::vector<Access>> hist;   // per buffer

  int add_buf(int kind, int node, int worker, uint64_t bytes) {
    PlanBuf b;
    b.kind = kind;
    b.node = node;
    b.worker = worker;
    b.bytes = bytes;
    P->bufs.push_back(b);
    hist.emplace_back();
    return static_cast<int>(P->bufs.size()) - 1;
  }

  struct Acc {
    int buf;
    int64_t off, ld, rows, cols;
    bool write;
  };

  void emit(northup_op op, std::initializer_list<Acc> accs) {
    const int idx = static_cast<int>(P->ops.size());
    // latest conflicting op per (worker, stream); ops on the op's own
    // (worker, stream) queue are ordered already.
    std::vector<std::pair<int, int>> last;   // (key, op)
    for (const Acc& a : accs) {
      if (a.rows <= 0 || a.cols <= 0) continue;
      const int64_t lo = a.off, hi = a.off + (a.rows - 1) * a.ld + a.cols;
      const bool user = P->bufs[a.buf].kind != B_ARENA && P->bufs[a.buf].kind != B_DRAM;
      auto& h = hist[a.buf];
      for (const Access& p : h) {
        if (!a.write && !p.write) continue;
        if (!overlaps(p, lo, hi, a.off, a.ld, a.rows, a.cols)) continue;
        const northup_op& q = P->ops[p.op];
        if (q.worker == op.worker && q.stream == op.stream) continue;
        // root-tier regions of different siblings are disjoint by construction
        // (their 2-D bounding intervals may still overlap)
        if (user_disjoint && user && q.worker != op.worker && !is_io_stream(q.stream) && !is_io_stream(op.stream))
          continue;
        const int key = q.worker * S_KEYS + q.stream;
        bool found = false;
        for (auto& kv : last)
          if (kv.first == key) {
            kv.second = std::max(kv.second, p.op);
            found = true;
          }
        if (!found) last.emplace_back(key, p.op);
      }
      h.push_back(Access{idx, op.stream, lo, hi, a.off, a.ld, a.rows, a.cols, a.write});
    }
    op.ndeps = 0;
    for (auto& kv : last) {
      if (op.ndeps >= 16) {
        overflow = true;
        break;
      }
      op.deps[op.ndeps++] = kv.second;
    }
    P->ops.push_back(op);
    if (!replica.empty() && op.op == NU_OP_COPY && P->bufs[op.dst_buf].kind == B_USER_C &&
        P->bufs[op.src_buf].kind == B_ARENA)
      push_replicas(op);
  }
  bool overflow = false;

  // replicate_result (S§8(e)) carried by the plan: every drain of a finished C
  // piece from a sibling's HBM to the root is followed by copies of the same
  // HBM region into every sibling's replica (peers first, its own last) on that
  // sibling's device-to-device stream, so the NVLink transfers overlap the
  // compute and drains still to come instead of running after the join.
  // replica[w] = plan buffer of sibling w's replica (M x N, ld = the root C's).
  std::vector<int> replica;
  void push_replicas(const northup_op& d) {
    const int G = static_cast<int>(replica.size());
    for (int k = 1; k <= G; ++k) {
      const int q = (d.worker + k) % G;
      emit(make_copy(d.worker, S_D2D, d.src_buf, d.src_off, d.src_ld, replica[q], d.dst_off, d.dst_ld, d.rows, d.cols),
           {{d.src_buf, d.src_off, d.src_ld, d.rows, d.cols, false}, {replica[q], d.dst_off, d.dst_ld, d.rows, d.cols, true}});
      P->stats.bytes_d2d += 4ull * d.rows * d.cols;
    }
  }
};



}  // namespace nu
