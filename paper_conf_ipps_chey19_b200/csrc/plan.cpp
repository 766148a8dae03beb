// Planner: the recursive decomposition of §IV-A over the Northup
// tree, unrolled into a per-GPU list of operations (Listing 3 P:204-221 with
// the recursion depth fixed by the tree).
//
//   level l (root, pinned host)  --data_down-->  level l+1 (HBM of GPU w)
//   level l+1 (HBM)              --TMA------->   SMEM/TMEM leaf (the kernel)
//
// Each op is COPY (data_down / data_up over PCIe), LEAF (compute_task at the
// leaf, accumulating partial sums) or ZERO.  Dependencies between ops
// are derived here from the byte ranges each op reads and writes, so the
// executor only has to turn them into CUDA stream waits.
//
// Schedules at the HOST -> HBM edge:
//   S2  C block resident in HBM, K panels of A and B stream through a ring of
//       kSlots slots; the last `tail_k` of K is computed strip by strip with a
//       resident B tail so each finished C strip drains (D2H) while the next
//       strip computes ("staggered drain").
//   S1  paper-literal row-shard reuse: row shard m of A stays in HBM
//       while the column shards of B stream; each C block drains when done.
#include <stdlib.h>
#include <algorithm>
#include <cmath>

#include "northup_internal.h"
#include "plan_builder.h"

namespace nu {


// Nominal planning constants: the leaf's useful flop rate on
// one B200 under its power cap (x3 leaf, measured 390 TF/s in-HBM on 32768^3)
// and the PCIe Gen5 x16 per-direction bandwidth measured with both directions
// busy (49-50 GB/s).  Only used to size the drain tail.
static constexpr double kPlanFlops = 390e12;
static constexpr double kPlanPcie = 49e9;

int partition_grid(int G, int64_t M, int64_t N, int* Pr, int* Pc) {
  if (G <= 0) return fail(NU_EINVAL, "G must be positive");
  int best_r = 1, best_c = G;
  int64_t best = -1;
  for (int r = 1; r <= G; ++r) {
    if (G % r) continue;
    const int c = G / r;
    // per-GPU H2D bytes ~ 4K (M/Pr + N/Pc); ties go to more row splits so
    // C regions stay contiguous in the row-major root.
    const int64_t cost = cdiv(M, r) + cdiv(N, c);
    if (best < 0 || cost < best || (cost == best && r > best_r)) {
      best = cost;
      best_r = r;
      best_c = c;
    }
  }
  *Pr = best_r;
  *Pc = best_c;
  return 0;
}

static void split_range(int64_t n, int parts, int i, int64_t* lo, int64_t* hi) {
  const int64_t step = cdiv(n, parts);
  *lo = std::min<int64_t>(n, step * i);
  *hi = std::min<int64_t>(n, *lo + step);
}

int region_of(int G, int64_t M, int64_t N, int r, int64_t* r0, int64_t* r1, int64_t* c0,
              int64_t* c1) {
  int Pr = 1, Pc = 1;
  int rc = partition_grid(G, M, N, &Pr, &Pc);
  if (rc) return rc;
  if (r < 0 || r >= G) return fail(NU_EINVAL, "region index out of range");
  split_range(M, Pr, r / Pc, r0, r1);
  split_range(N, Pc, r % Pc, c0, c1);
  return 0;
}

// The leaf scratch of worker w: the last `scr` bytes of its arena buffer.
static void set_scratch(Plan* P, int w, int buf, uint64_t arena_bytes, uint64_t scr) {
  if (static_cast<int>(P->scr_buf.size()) <= w) {
    P->scr_buf.resize(w + 1, -1);
    P->scr_off.resize(w + 1, 0);
    P->scr_bytes.resize(w + 1, 0);
  }
  P->scr_buf[w] = buf;
  P->scr_off[w] = arena_bytes - scr;
  P->scr_bytes[w] = scr;
}

namespace {

northup_op make_leaf(int worker, int a, int64_t a_off, int64_t lda, int b, int64_t b_off,
                     int64_t ldb, int c, int64_t c_off, int64_t ldc, int64_t m, int64_t n, int64_t k,
                     int accumulate) {
  northup_op o{};
  o.op = NU_OP_LEAF;
  o.worker = worker;
  o.stream = S_COMP;
  o.a_buf = a;
  o.b_buf = b;
  o.c_buf = c;
  o.a_off = a_off;
  o.b_off = b_off;
  o.c_off = c_off;
  o.lda = lda;
  o.ldb = ldb;
  o.ldc = ldc;
  o.m = m;
  o.n = n;
  o.k = k;
  o.accumulate = accumulate;
  o.src_buf = o.dst_buf = -1;
  return o;
}

// In-place split of a resident B region (one K panel: rows x cols at off, ld),
// column exponents to (ebuf, eoff).  Runs on the compute stream, in order with
// the leaf ops that use the worker's scratch.
northup_op make_split_b(int worker, int buf, int64_t off, int64_t ld, int64_t rows, int64_t cols, int ebuf,
                        int64_t eoff) {
  northup_op o{};
  o.op = NU_OP_SPLIT_B;
  o.worker = worker;
  o.stream = S_COMP;
  o.dst_buf = buf;
  o.dst_off = off;
  o.dst_ld = ld;
  o.rows = rows;
  o.cols = cols;
  o.c_buf = ebuf;
  o.c_off = eoff;
  o.src_buf = o.a_buf = o.b_buf = -1;
  return o;
}

// Mark a leaf op as reading a pre-split B (exponents at ebuf/eoff, `stride`
// per K panel).
northup_op with_presplit_b(northup_op o, int ebuf, int64_t eoff, int64_t stride) {
  o.src_buf = ebuf;
  o.src_off = eoff;
  o.rows = stride;
  return o;
}

struct EdgeCtx {
  Builder* B;
  int worker;
  int hbm_node;
  int A, Bb, C;            // user buffers (root tier)
  int64_t lda, ldb, ldc;   // root leading dims
  int64_t r0, r1, c0, c1;  // region
  int64_t K;
  uint64_t cap;            // HBM capacity (bytes)
  int64_t kc;
  int64_t obm, obn, obk;   // block override at the parent node
  int sched;
  // NVLink-shared staging (S§8(f) NEXT-1): this worker loads 1/a_share of each
  // A panel and 1/b_share of each B panel over PCIe, its row / column peers
  // the rest, and pulls the other pieces from them over NVLink.
  int a_share = 1, b_share = 1;
  double pcie = 0.0;       // B/s per GPU measured at finalize (0: kPlanPcie)
  // S2's B-first variant: 0 = the cost model picks between it
  // and the drain-tail schedule, -1 = never (NU_SCHED_S2, shared staging),
  // 1 = whenever it fits (NU_SCHED_S2B).
  int bfirst = 0;
  // Origin of the region in the root buffers' addressing: (r0, c0) for a
  // whole-problem root; (0, 0) with ldb = ldc = region width when the root
  // buffers hold only this sibling's strips (multi-process siblings).
  int64_t ar0 = 0, ac0 = 0;
};

// ---------------------------------------------------------------- S2
struct S2Shape {
  int64_t bm, bn, bk, tail, sr;
  uint64_t bytes;
  int64_t r1 = 0;   // > 0: B-first — rows [0, r1) of the block in the main phase (tail = K)
};

uint64_t s2_bytes(int64_t bm, int64_t bn, int64_t bk, int64_t K, int64_t tail, int64_t sr, int64_t kc) {
  const int64_t kmain = K - tail;
  uint64_t e = static_cast<uint64_t>(bm) * pad_ld(bn);                    // C block
  if (kmain > 0)
    e += static_cast<uint64_t>(kSlots) *
         (static_cast<uint64_t>(bm) * pad_ld(bk) + static_cast<uint64_t>(bk) * pad_ld(bn));
  if (tail > 0)
    e += static_cast<uint64_t>(rup(tail, 32)) * pad_ld(bn) +                 // B tail (split in place)
         static_cast<uint64_t>(kSlots) * sr * pad_ld(tail) +                 // A strips
         static_cast<uint64_t>(cdiv(tail, kc)) * pad_ld(bn);                 // B tail column exponents
  return e * 4 + leaf_scratch(bm, bn, kc);                                   // + leaf scratch
}

// Predicted time of one S2 block with drain tail K_t: the main
// phase streams the A/B panels of K - K_t plus the resident B tail over H2D
// while computing K - K_t; the tail phase computes row strips over K_t while
// their A strips arrive (H2D) and finished C strips leave (D2H).
// With shared staging only this worker's pieces (1/a_share of A, 1/b_share of
// B) cross its PCIe link; NVLink pulls are ~20x faster and not modelled.
static double s2_time(int64_t bm, int64_t bn, int64_t K, int64_t tail, int a_share, int b_share,
                      double pcie) {
  const double kPlanPcie = pcie > 0 ? pcie : nu::kPlanPcie;   // measured at finalize when available
  const double fl = 2.0 * bm * bn / kPlanFlops;               // s per unit of K
  const double ea = static_cast<double>(bm) / a_share, eb = static_cast<double>(bn) / b_share;
  const double main_c = fl * (K - tail);
  const double main_h = 4.0 * ((ea + eb) * static_cast<double>(K - tail) + static_cast<double>(tail) * eb) /
                        kPlanPcie;
  const double tail_c = fl * tail;
  const double tail_h = 4.0 * ea * static_cast<double>(tail) / kPlanPcie;
  const double d2h = 4.0 * bm * static_cast<double>(bn) / kPlanPcie;
  return std::max(main_c, main_h) + std::max(std::max(tail_c, tail_h), d2h);
}

// ------------------------------------------------ S2, B-first variant
// Under S2 a C row is final only after its last K panel, so C's D2H overlaps
// only the tail phase (the "structural bound").  The B-first
// variant keeps ALL of B resident (split once, in place, as it lands): while
// B's K panels stream in, rows [0, r1) of the block are computed panel by
// panel (their A panels through kSlots slots); then the other rows run as
// strips over the full K against the resident B, and the r1 finished rows
// drain while those strips compute.  Arena (elements):
//   [C rows r1 x pad(bn)] [kSlots x A slot r1 x pad(bk)] [B K x pad(bn)]
//   [kSlots x A strip sr x pad(K)] [kSlots x C strip sr x pad(bn)]
//   [B column exponents: one row of pad(bn) ints per K panel] [leaf scratch]
uint64_t bfirst_bytes(int64_t r1, int64_t bn, int64_t bk, int64_t K, int64_t sr, int64_t kc) {
  uint64_t e = static_cast<uint64_t>(r1) * pad_ld(bn) + static_cast<uint64_t>(kSlots) * r1 * pad_ld(bk) +
               static_cast<uint64_t>(rup(K, 32)) * pad_ld(bn) +
               static_cast<uint64_t>(kSlots) * sr * (pad_ld(K) + pad_ld(bn)) +
               static_cast<uint64_t>(cdiv(K, kc)) * pad_ld(bn);
  return e * 4 + leaf_scratch(std::max(r1, sr), bn, kc);
}

// Predicted block time (same rates as s2_time): phase 1 = max(compute of r1
// rows, H2D of B + their A), phase 2 = max(compute of the other rows, H2D of
// their A, D2H of the whole block), plus the fill before the first leaf (one
// B panel and a quarter of an A panel).
static double bfirst_time(int64_t bm, int64_t bn, int64_t K, int64_t r1, int64_t kc, double pcie) {
  const double bw = pcie > 0 ? pcie : nu::kPlanPcie;
  const double fl = 2.0 * static_cast<double>(bn) * K / kPlanFlops;   // s per C row
  const double row_h = 4.0 * K / bw;                                   // A row, s
  const double p1 = std::max(fl * r1, 4.0 * static_cast<double>(bn) * K / bw + row_h * r1);
  const double p2 = std::max(std::max(fl * (bm - r1), row_h * (bm - r1)), 4.0 * bm * static_cast<double>(bn) / bw);
  return p1 + p2 + 4.0 * (bn + r1 / 4.0) * kc / bw;
}

int choose_s2(const EdgeCtx& x, S2Shape* out) {
  const int64_t m = x.r1 - x.r0, n = x.c1 - x.c0, K = x.K;
  const uint64_t cap = x.cap ? x.cap : (uint64_t(1) << 62);
  int64_t bk = x.obk > 0 ? x.obk : std::max<int64_t>(x.kc, 4);
  bk = std::min<int64_t>(bk, rup(K, 4));
  std::vector<int64_t> bms, bns;
  int64_t bm0 = x.obm > 0 ? std::min(x.obm, m) : m;
  int64_t bn0 = x.obn > 0 ? std::min(x.obn, n) : n;
  for (int64_t v = bm0;; v = rup(cdiv(v, 2), 128)) {
    bms.push_back(v);
    if (v <= 128) break;
  }
  for (int64_t v = bn0;; v = rup(cdiv(v, 2), 256)) {
    bns.push_back(v);
    if (v <= 256) break;
  }
  // drain-tail candidates: multiples of k_chunk (at most ~64 of them) and K
  std::vector<int64_t> tails{0};
  const int64_t tstep = std::max<int64_t>(x.kc, rup(cdiv(K, 64), x.kc));
  for (int64_t t = tstep; t < K; t += tstep) tails.push_back(t);
  tails.push_back(K);
  // Among the C-block shapes that fit, pick the fewest H2D bytes: every block
  // streams its A row strip and B column strip once, 4K(bm + bn) per block.
  // For each shape the drain tail minimises the predicted block time (ties:
  // the longer tail); ties between shapes: predicted time, then taller blocks
  // (contiguous C rows in the root).
  bool found = false;
  S2Shape best{};
  uint64_t best_h2d = 0;
  double best_t = 0;
  for (int64_t bn : bns) {
    for (int64_t bm : bms) {
      // per-GPU PCIe bytes per unit of K, scaled by a_share * b_share (shared
      // staging divides A by a_share and B by b_share)
      const uint64_t h2d = static_cast<uint64_t>(cdiv(m, bm) * cdiv(n, bn)) *
                           static_cast<uint64_t>(bm * x.b_share + bn * x.a_share);
      if (found && h2d > best_h2d) continue;
      const int64_t strips = std::max<int64_t>(1, std::min<int64_t>(16, cdiv(bm, 1024)));
      const int64_t sr = std::min(rup(cdiv(bm, strips), 128), bm);
      bool have = false;
      S2Shape cand{};
      double cand_t = 0;
      for (int64_t tail : tails) {
        uint64_t bytes = s2_bytes(bm, bn, bk, K, tail, sr, x.kc);
        int64_t use_bk = bk;
        if (bytes > cap && tail == 0 && bk > x.kc && x.obk <= 0) {   // the minimum panel
          use_bk = x.kc;
          bytes = s2_bytes(bm, bn, use_bk, K, 0, 0, x.kc);
        }
        if (bytes > cap) continue;
        const double t = s2_time(bm, bn, K, tail, x.a_share, x.b_share, x.pcie);
        if (!have || t <= cand_t * (1.0 + 1e-9)) {
          cand = S2Shape{bm, bn, use_bk, tail, tail > 0 ? sr : 0, bytes};
          cand_t = t;
          have = true;
        }
      }
      if (have && x.bfirst >= 0) {
        // compare with the B-first variant, both with their pipeline fill (the
        // drain-tail schedule computes its first panel on a 4 x 4 sub-grid)
        const double bw = x.pcie > 0 ? x.pcie : kPlanPcie;
        double best_b = cand_t + 4.0 * (bm + bn) / 4.0 * bk / bw;
        if (x.bfirst > 0) best_b = 1e300;
        S2Shape bc{};
        bool have_b = false;
        // Needs a pre-split B (<= kLeafMaxN columns).  The model considers it
        // only for a region that is ONE block, with at least two K panels and
        // the caller's K panel: with several blocks the drain-tail S2 already
        // overlaps one block's D2H-bound tail with the next block's H2D-bound
        // main phase (measured: cfg4 on one GPU 340 vs 334 TF/s, cfg5 94 vs 81),
        // while B-first blocks serialise on the shared resident B.
        const bool one_block = bm >= m && bn >= n;
        if (bn <= kLeafMaxN && bm >= 2 && (x.bfirst > 0 || (one_block && K > x.kc && x.obk <= 0))) {
          const int64_t step = std::max<int64_t>(128, rup(cdiv(bm, 64), 128));
          const int64_t sr2 = std::max<int64_t>(1, std::min<int64_t>(1024, rup(cdiv(bm, 32), 128)));
          for (int64_t r1 = std::min(step, bm - 1); r1 < bm; r1 += step) {
            const uint64_t bytes = bfirst_bytes(r1, bn, x.kc, K, sr2, x.kc);
            if (bytes > cap) break;
            const double t = bfirst_time(bm, bn, K, r1, x.kc, x.pcie);
            if (t < best_b * (1.0 - 1e-9)) {
              best_b = t;
              bc = S2Shape{bm, bn, x.kc, K, sr2, bytes, r1};
              have_b = true;
            }
          }
        }
        if (have_b) {
          cand = bc;
          cand_t = best_b;
        }
      }
      if (!have) continue;
      const double tot = cand_t * static_cast<double>(cdiv(m, bm) * cdiv(n, bn));
      const bool better = !found || h2d < best_h2d || (h2d == best_h2d && tot < best_t * (1.0 - 1e-9)) ||
                          (h2d == best_h2d && tot <= best_t * (1.0 + 1e-9) && bm > best.bm);
      if (better) {
        best = cand;
        best_h2d = h2d;
        best_t = tot;
        found = true;
      }
    }
  }
  // Whole-region B-first when the drain-tail S2 needs several C blocks but
  // all of B fits beside a few strips (tall-skinny regions such as cfg5): one
  // pass over A with B resident, every C strip drained as soon as it is done,
  // so H2D (A) and D2H (C) run concurrently from start to end.  The
  // multi-block drain-tail estimate counts its blocks as pipelined (a block's
  // tail overlaps the next block's loads) plus half a block's drain at the end.
  if (found && x.bfirst >= 0 && best.r1 == 0 && (best.bm < m || best.bn < n) && n <= kLeafMaxN && K > x.kc &&
      x.obk <= 0) {
    const double bw = x.pcie > 0 ? x.pcie : kPlanPcie;
    const double nb = static_cast<double>(cdiv(m, best.bm) * cdiv(n, best.bn));
    const double blk_c = 2.0 * best.bm * best.bn * static_cast<double>(K) / kPlanFlops;
    const double blk_h = 4.0 * static_cast<double>(best.bm + best.bn) * K / bw;
    const double blk_d = 4.0 * static_cast<double>(best.bm) * best.bn / bw;
    const double classic = nb * std::max(blk_c, std::max(blk_h, blk_d)) + blk_d / 2;
    const int64_t sr2 = std::min<int64_t>(8192, std::max<int64_t>(128, rup(cdiv(m, 128), 128)));
    const int64_t step = std::max<int64_t>(128, rup(cdiv(m, 64), 128));
    double best_b = x.bfirst > 0 ? 1e300 : classic;
    S2Shape bc{};
    bool have_b = false;
    for (int64_t r1 = std::min(step, m - 1); r1 < m && r1 > 0; r1 += step) {
      const uint64_t bytes = bfirst_bytes(r1, n, x.kc, K, sr2, x.kc);
      if (bytes > cap) break;
      const double t = bfirst_time(m, n, K, r1, x.kc, x.pcie);
      if (t < best_b * (1.0 - 1e-9)) {
        best_b = t;
        bc = S2Shape{m, n, x.kc, K, sr2, bytes, r1};
        have_b = true;
      }
    }
    if (have_b) best = bc;
  }
  if (found) {
    *out = best;
    return 0;
  }
  return fail(NU_ENOMEM, "HBM node %d capacity %llu B is below the minimum block", x.hbm_node,
              (unsigned long long)x.cap);
}

// Arena layout of one S2 worker (elements):
//   [C block bm x pad(bn)] [kSlots x (A slot bm x pad(bk), B slot bk x pad(bn))]
//   [B tail tail x pad(bn)] [kSlots x A strip sr x pad(tail)]
struct S2Layout {
  int arena = -1;
  int64_t ldC = 0, ldA = 0, ldBs = 0, ldAt = 0;
  int64_t offC = 0, offBT = 0;
  int64_t offEB = -1;   // B tail column exponents [panel][ldBs] (ints), when the tail is split in place
  int64_t offSA[kSlots] = {}, offSB[kSlots] = {}, offAT[kSlots] = {};
  int64_t offCS[kSlots] = {};   // B-first: C strip slots
};

S2Layout layout_s2(Builder& B, const S2Shape& s, int hbm_node, int w, int64_t K) {
  S2Layout L;
  L.arena = B.add_buf(B_ARENA, hbm_node, w, s.bytes);
  if (s.r1 > 0) {   // B-first (see bfirst_bytes)
    set_scratch(B.P, w, L.arena, s.bytes, leaf_scratch(std::max(s.r1, s.sr), s.bn, B.P->kc));
    L.ldC = L.ldBs = pad_ld(s.bn);
    L.ldA = pad_ld(s.bk);
    L.ldAt = pad_ld(K);
    int64_t off = 0;
    L.offC = off;
    off += s.r1 * L.ldC;
    for (int i = 0; i < kSlots; ++i, off += s.r1 * L.ldA) L.offSA[i] = off;
    L.offBT = off;
    off += rup(K, 32) * L.ldBs;
    for (int i = 0; i < kSlots; ++i, off += s.sr * L.ldAt) L.offAT[i] = off;
    for (int i = 0; i < kSlots; ++i, off += s.sr * L.ldC) L.offCS[i] = off;
    L.offEB = off;
    return L;
  }
  set_scratch(B.P, w, L.arena, s.bytes, leaf_scratch(s.bm, s.bn, B.P->kc));
  L.ldC = pad_ld(s.bn);
  L.ldA = pad_ld(s.bk);
  L.ldBs = pad_ld(s.bn);
  L.ldAt = pad_ld(s.tail);
  int64_t off = 0;
  L.offC = off;
  off += s.bm * L.ldC;
  const int64_t kmain = K - s.tail;
  for (int i = 0; i < kSlots; ++i) {
    L.offSA[i] = off;
    off += kmain > 0 ? s.bm * L.ldA : 0;
    L.offSB[i] = off;
    off += kmain > 0 ? s.bk * L.ldBs : 0;
  }
  if (s.tail > 0) {
    L.offBT = off;
    off += rup(s.tail, 32) * L.ldBs;
    for (int i = 0; i < kSlots; ++i) {
      L.offAT[i] = off;
      off += s.sr * L.ldAt;
    }
    if (s.bn <= kLeafMaxN) L.offEB = off;   // wider tails are split by each leaf call instead
    off += cdiv(s.tail, B.P->kc) * L.ldBs;
  }
  return L;
}

// The B tail is resident for the whole tail phase and read by every strip's
// leaf: split each loaded piece (one K panel) once, in place, instead of in
// every leaf call (R22).  Pieces are bk = k_chunk rows.
void emit_tail_split(Builder& B, int w, const S2Layout& L, const S2Shape& s, int64_t bn, int64_t kt0,
                     int64_t kk) {
  if (L.offEB < 0) return;
  const int64_t kc = B.P->kc, p = kt0 / kc;
  for (int64_t k = kt0; k < kt0 + kk; k += kc) {   // a piece is a whole number of panels
    const int64_t rows = std::min(kc, kt0 + kk - k), pp = k / kc;
    (void)p;
    // the split form of an n-column row occupies hi at elements [0, n/2) and lo
    // at [ld/2, ld/2 + n/2) of the row: declare the whole row (n < ld for a
    // ragged last block)
    B.emit(make_split_b(w, L.arena, L.offBT + k * L.ldBs, L.ldBs, rows, bn, L.arena, L.offEB + pp * L.ldBs),
           {{L.arena, L.offBT + k * L.ldBs, L.ldBs, rup(rows, 32), L.ldBs, true},
            {L.arena, L.offEB + pp * L.ldBs, L.ldBs, 1, bn, true}});
  }
}

void emit_tail_leaf(Builder& B, int w, const S2Layout& L, const S2Shape& s, int ar, int64_t ao, int64_t lda,
                    int64_t co, int64_t ldc, int64_t rr, int64_t bn, int acc) {
  northup_op o = make_leaf(w, ar, ao, lda, L.arena, L.offBT, L.ldBs, ar, co, ldc, rr, bn, s.tail, acc);
  if (L.offEB >= 0) {
    o = with_presplit_b(o, L.arena, L.offEB, L.ldBs);
    B.emit(o, {{ar, ao, lda, rr, s.tail, false},
               {L.arena, L.offBT, L.ldBs, s.tail, L.ldBs, false},     // the split rows' full span
               {L.arena, L.offEB, L.ldBs, cdiv(s.tail, B.P->kc), bn, false},
               {ar, co, ldc, rr, bn, true}});
  } else {
    B.emit(o, {{ar, ao, lda, rr, s.tail, false}, {L.arena, L.offBT, L.ldBs, s.tail, bn, false},
               {ar, co, ldc, rr, bn, true}});
  }
}

// Rows of the graded drain strips (full strips while more than two remain,
// then halving sizes, so the last D2H is small).
// Never more than sr rows: a strip must fit its slot.
static int64_t next_strip(int64_t bm, int64_t r, int64_t sr) {
  const int64_t rem = bm - r;
  if (rem > 2 * sr) return sr;
  if (rem <= std::min<int64_t>(512, sr)) return rem;
  return std::min(sr, rup(cdiv(rem, 2), 128));
}

void s2_stats(const S2Shape& s, northup_stats* st) {
  st->bm = s.bm;
  st->bn = s.bn;
  st->bk = s.bk;
  st->tail_k = s.tail;
  st->strips = 0;
  for (int64_t r = s.r1; s.tail > 0 && r < s.bm; r += next_strip(s.bm, r, s.sr), ++st->strips) {
  }
  st->hbm_peak_bytes = s.bytes;
  st->schedule = s.r1 > 0 ? NU_SCHED_S2B : NU_SCHED_S2;
  st->bfirst_rows = static_cast<int>(s.r1);
}

// One C block (rows gr.., cols gc.., bm x bn) under the B-first variant.
static void emit_bfirst_block(const EdgeCtx& x, const S2Shape& s, const S2Layout& L, int64_t gr, int64_t gc,
                              int64_t bm, int64_t bn, int* panel_it, int* strip_it, northup_stats* st) {
  Builder& B = *x.B;
  const int w = x.worker, arena = L.arena;
  const int64_t K = x.K, kc = B.P->kc, r1 = std::min(s.r1, bm);
  const int64_t ldC = L.ldC, ldA = L.ldA, ldBs = L.ldBs, ldAt = L.ldAt;
  const bool presplit = bn <= kLeafMaxN;
  // ---- phase 1: B's K panels land in the resident B and rows [0, r1) accumulate
  const int64_t npan = cdiv(K, kc);
  for (int64_t p = 0; p < npan; ++p, ++*panel_it) {
    const int sl = *panel_it % kSlots;
    const int64_t k0 = p * kc, kk = std::min(kc, K - k0);
    const int64_t boff = L.offBT + k0 * ldBs, eoff = L.offEB + p * ldBs;
    // Panel 0 gates the pipeline fill: it is computed on a 4 x 4 sub-grid from
    // the raw B (each leaf splits its piece) and split in place afterwards, so
    // the first leaf waits for a quarter of the panel instead of all of it.
    const int64_t gb = (p == 0 && r1 >= 4096 && bn >= 4096) ? 4 : 1;
    const int64_t sbm = rup(cdiv(r1, gb), 256), sbn = rup(cdiv(bn, gb), 256);
    for (int64_t jj = 0; jj < bn; jj += sbn) {
      const int64_t cn = std::min(sbn, bn - jj);
      B.emit(make_copy(w, S_H2D, x.Bb, k0 * x.ldb + gc + jj, x.ldb, arena, boff + jj, ldBs, kk, cn),
             {{x.Bb, k0 * x.ldb + gc + jj, x.ldb, kk, cn, false}, {arena, boff + jj, ldBs, kk, cn, true}});
      st->bytes_h2d += static_cast<uint64_t>(kk) * cn * 4;
      if (gb == 1 && presplit)   // the whole panel row span is loaded: split it in place
        B.emit(make_split_b(w, arena, boff, ldBs, kk, bn, arena, eoff),
               {{arena, boff, ldBs, rup(kk, 32), ldBs, true}, {arena, eoff, ldBs, 1, bn, true}});
      for (int64_t ii = 0; ii < r1; ii += sbm) {
        const int64_t rm = std::min(sbm, r1 - ii);
        if (jj == 0) {
          B.emit(make_copy(w, S_H2D, x.A, (gr + ii) * x.lda + k0, x.lda, arena, L.offSA[sl] + ii * ldA, ldA, rm,
                           kk),
                 {{x.A, (gr + ii) * x.lda + k0, x.lda, rm, kk, false},
                  {arena, L.offSA[sl] + ii * ldA, ldA, rm, kk, true}});
          st->bytes_h2d += static_cast<uint64_t>(rm) * kk * 4;
        }
        northup_op o = make_leaf(w, arena, L.offSA[sl] + ii * ldA, ldA, arena, boff + jj, ldBs, arena,
                                 L.offC + ii * ldC + jj, ldC, rm, cn, kk, p > 0 ? 1 : 0);
        if (gb == 1 && presplit) {
          o = with_presplit_b(o, arena, eoff, ldBs);
          B.emit(o, {{arena, L.offSA[sl] + ii * ldA, ldA, rm, kk, false},
                     {arena, boff, ldBs, kk, ldBs, false},
                     {arena, eoff, ldBs, 1, bn, false},
                     {arena, L.offC + ii * ldC + jj, ldC, rm, cn, true}});
        } else {
          B.emit(o, {{arena, L.offSA[sl] + ii * ldA, ldA, rm, kk, false},
                     {arena, boff + jj, ldBs, kk, cn, false},
                     {arena, L.offC + ii * ldC + jj, ldC, rm, cn, true}});
        }
        st->leaf_launches++;
      }
    }
    if (gb > 1 && presplit)   // panel 0 after its sub-grid leaves
      B.emit(make_split_b(w, arena, boff, ldBs, kk, bn, arena, eoff),
             {{arena, boff, ldBs, rup(kk, 32), ldBs, true}, {arena, eoff, ldBs, 1, bn, true}});
  }
  // ---- phase 2: the other rows as strips over the full K against the resident
  // B, while rows [0, r1) drain (one piece before each strip's own D2H)
  int64_t nstrips = 0;
  for (int64_t r = r1; r < bm; r += next_strip(bm, r, s.sr)) ++nstrips;
  const int64_t piece = nstrips > 0 ? cdiv(r1, nstrips) : r1;
  int64_t drained = 0;
  auto drain_piece = [&]() {
    const int64_t rr = std::min(piece, r1 - drained);
    if (rr <= 0) return;
    B.emit(make_copy(w, S_D2H, arena, L.offC + drained * ldC, ldC, x.C, (gr + drained) * x.ldc + gc, x.ldc, rr, bn),
           {{arena, L.offC + drained * ldC, ldC, rr, bn, false},
            {x.C, (gr + drained) * x.ldc + gc, x.ldc, rr, bn, true}});
    st->bytes_d2h += static_cast<uint64_t>(rr) * bn * 4;
    drained += rr;
  };
  for (int64_t r = r1, rr = 0; r < bm; r += rr, ++*strip_it) {
    rr = next_strip(bm, r, s.sr);
    const int sl = *strip_it % kSlots;
    B.emit(make_copy(w, S_H2D, x.A, (gr + r) * x.lda, x.lda, arena, L.offAT[sl], ldAt, rr, K),
           {{x.A, (gr + r) * x.lda, x.lda, rr, K, false}, {arena, L.offAT[sl], ldAt, rr, K, true}});
    st->bytes_h2d += static_cast<uint64_t>(rr) * K * 4;
    northup_op o = make_leaf(w, arena, L.offAT[sl], ldAt, arena, L.offBT, ldBs, arena, L.offCS[sl], ldC, rr, bn, K, 0);
    if (presplit) {
      o = with_presplit_b(o, arena, L.offEB, ldBs);
      B.emit(o, {{arena, L.offAT[sl], ldAt, rr, K, false},
                 {arena, L.offBT, ldBs, K, ldBs, false},
                 {arena, L.offEB, ldBs, cdiv(K, kc), bn, false},
                 {arena, L.offCS[sl], ldC, rr, bn, true}});
    } else {
      B.emit(o, {{arena, L.offAT[sl], ldAt, rr, K, false},
                 {arena, L.offBT, ldBs, K, bn, false},
                 {arena, L.offCS[sl], ldC, rr, bn, true}});
    }
    st->leaf_launches++;
    drain_piece();
    B.emit(make_copy(w, S_D2H, arena, L.offCS[sl], ldC, x.C, (gr + r) * x.ldc + gc, x.ldc, rr, bn),
           {{arena, L.offCS[sl], ldC, rr, bn, false}, {x.C, (gr + r) * x.ldc + gc, x.ldc, rr, bn, true}});
    st->bytes_d2h += static_cast<uint64_t>(rr) * bn * 4;
  }
  while (drained < r1) drain_piece();
}

int build_s2(const EdgeCtx& x, northup_stats* st) {
  S2Shape s{};
  int rc = choose_s2(x, &s);
  if (rc) return rc;
  Builder& B = *x.B;
  const int w = x.worker;
  const int64_t m = x.r1 - x.r0, n = x.c1 - x.c0, K = x.K;
  const S2Layout L = layout_s2(B, s, x.hbm_node, w, K);
  const int arena = L.arena;
  const int64_t ldC = L.ldC, ldA = L.ldA, ldBs = L.ldBs, ldAt = L.ldAt, offC = L.offC, offBT = L.offBT;
  const int64_t* offSA = L.offSA;
  const int64_t* offSB = L.offSB;
  const int64_t* offAT = L.offAT;
  const int64_t kmain = K - s.tail;
  if (w == 0) s2_stats(s, st);
  int panel_it = 0, strip_it = 0;
  for (int64_t i0 = 0; i0 < m; i0 += s.bm) {
    const int64_t bm = std::min(s.bm, m - i0);
    for (int64_t j0 = 0; j0 < n; j0 += s.bn) {
      const int64_t bn = std::min(s.bn, n - j0);
      const int64_t gr = x.ar0 + i0, gc = x.ac0 + j0;   // root row/col of the block
      if (s.r1 > 0) {
        emit_bfirst_block(x, s, L, gr, gc, bm, bn, &panel_it, &strip_it, st);
        continue;
      }
      // ---- main phase: K panels [0, kmain)
      const int64_t npan = kmain > 0 ? cdiv(kmain, s.bk) : 0;
      const int64_t ntail_pieces = s.tail > 0 ? cdiv(s.tail, s.bk) : 0;
      int64_t pieces_done = 0;
      auto load_tail_piece = [&](int64_t piece) {
        const int64_t k0 = kmain + piece * s.bk, kk = std::min(s.bk, K - k0);
        B.emit(make_copy(w, S_H2D, x.Bb, k0 * x.ldb + gc, x.ldb, arena, offBT + (k0 - kmain) * ldBs,
                         ldBs, kk, bn),
               {{x.Bb, k0 * x.ldb + gc, x.ldb, kk, bn, false},
                {arena, offBT + (k0 - kmain) * ldBs, ldBs, kk, bn, true}});
        st->bytes_h2d += static_cast<uint64_t>(kk) * bn * 4;
        emit_tail_split(B, w, L, s, bn, k0 - kmain, kk);
      };
      for (int64_t p = 0; p < npan; ++p, ++panel_it) {
        const int sl = panel_it % kSlots;
        const int64_t k0 = p * s.bk, kk = std::min(s.bk, kmain - k0);
        st->bytes_h2d += static_cast<uint64_t>(bm) * kk * 4 + static_cast<uint64_t>(kk) * bn * 4;
        // The first panel is computed in a 4 x 4 grid of sub-blocks so the
        // leaf starts after 1/4 of A's and B's panel have landed instead of
        // the whole panel (pipeline fill); per-element arithmetic is unchanged.
        const int64_t gb = (p == 0 && bm >= 4096 && bn >= 4096) ? 4 : 1;
        const int64_t sbm = rup(cdiv(bm, gb), 256), sbn = rup(cdiv(bn, gb), 256);
        for (int64_t jj = 0; jj < bn; jj += sbn) {
          const int64_t cn = std::min(sbn, bn - jj);
          B.emit(make_copy(w, S_H2D, x.Bb, k0 * x.ldb + gc + jj, x.ldb, arena, offSB[sl] + jj, ldBs,
                           kk, cn),
                 {{x.Bb, k0 * x.ldb + gc + jj, x.ldb, kk, cn, false},
                  {arena, offSB[sl] + jj, ldBs, kk, cn, true}});
          for (int64_t ii = 0; ii < bm; ii += sbm) {
            const int64_t rm = std::min(sbm, bm - ii);
            if (jj == 0)
              B.emit(make_copy(w, S_H2D, x.A, (gr + ii) * x.lda + k0, x.lda, arena,
                               offSA[sl] + ii * ldA, ldA, rm, kk),
                     {{x.A, (gr + ii) * x.lda + k0, x.lda, rm, kk, false},
                      {arena, offSA[sl] + ii * ldA, ldA, rm, kk, true}});
            B.emit(make_leaf(w, arena, offSA[sl] + ii * ldA, ldA, arena, offSB[sl] + jj, ldBs, arena,
                             offC + ii * ldC + jj, ldC, rm, cn, kk, p > 0 ? 1 : 0),
                   {{arena, offSA[sl] + ii * ldA, ldA, rm, kk, false},
                    {arena, offSB[sl] + jj, ldBs, kk, cn, false},
                    {arena, offC + ii * ldC + jj, ldC, rm, cn, true}});
            st->leaf_launches++;
          }
        }
        // interleave the B-tail pieces over the main phase so they overlap
        // compute; none during the first panels, whose copies gate the
        // pipeline fill (the H2D stream is in-order)
        const int64_t skip = std::min<int64_t>(2, std::max<int64_t>(0, npan - 1));
        while (pieces_done < ntail_pieces && p >= skip &&
               (pieces_done + 1) * (npan - skip) <= (p + 1 - skip) * ntail_pieces) {
          load_tail_piece(pieces_done++);
        }
      }
      while (pieces_done < ntail_pieces) load_tail_piece(pieces_done++);
      if (s.tail > 0) {
        // ---- tail phase: strips of C finish and drain one by one
        // Graded strips: full strips while more than two remain, then halving
        // sizes, so the last D2H (the exposed drain) is small.
        for (int64_t r = 0, rr = 0; r < bm; r += rr, ++strip_it) {
          rr = next_strip(bm, r, s.sr);
          const int sl = strip_it % kSlots;
          B.emit(make_copy(w, S_H2D, x.A, (gr + r) * x.lda + kmain, x.lda, arena, offAT[sl], ldAt, rr,
                           s.tail),
                 {{x.A, (gr + r) * x.lda + kmain, x.lda, rr, s.tail, false},
                  {arena, offAT[sl], ldAt, rr, s.tail, true}});
          st->bytes_h2d += static_cast<uint64_t>(rr) * s.tail * 4;
          emit_tail_leaf(B, w, L, s, arena, offAT[sl], ldAt, offC + r * ldC, ldC, rr, bn, kmain > 0 ? 1 : 0);
          st->leaf_launches++;
          B.emit(make_copy(w, S_D2H, arena, offC + r * ldC, ldC, x.C, (gr + r) * x.ldc + gc, x.ldc, rr,
                           bn),
                 {{arena, offC + r * ldC, ldC, rr, bn, false},
                  {x.C, (gr + r) * x.ldc + gc, x.ldc, rr, bn, true}});
          st->bytes_d2h += static_cast<uint64_t>(rr) * bn * 4;
        }
      } else {
        B.emit(make_copy(w, S_D2H, arena, offC, ldC, x.C, gr * x.ldc + gc, x.ldc, bm, bn),
               {{arena, offC, ldC, bm, bn, false}, {x.C, gr * x.ldc + gc, x.ldc, bm, bn, true}});
        st->bytes_d2h += static_cast<uint64_t>(bm) * bn * 4;
      }
    }
  }
  return 0;
}

// ------------------------------------------- S2 with NVLink-shared staging
// S§8(f) NEXT-1 (P:230 siblings; "streaming over networks").  The G
// siblings form the partition grid Pr x Pc: the Pc siblings of a grid row need
// the same A panels, the Pr siblings of a grid column the same B panels.  Per
// K panel every sibling loads only its piece over its own PCIe link (rows
// piece j of the A panel, j = its index in the grid row; columns piece i of the
// B panel, i = its index in the grid column) and pulls the other pieces from
// its peers' HBM slots with a copy on its own D2D stream (NVLink P2P between
// devices, a local copy between virtual siblings of one device).  All workers
// use the same S2 shape and arena layout; the plan is emitted in lock step
// (loads, then pulls, then leaves of a panel, for all workers) so every pull's
// cross-worker dependency points backwards in plan order.  The leaf ops and
// their K-panel sequence are those of build_s2, so C is bitwise identical.
static void piece_range(int64_t n, int parts, int q, int64_t* lo, int64_t* hi) {
  const int64_t step = rup(cdiv(n, parts), 32);   // 128-B aligned piece edges
  *lo = std::min(n, step * q);
  *hi = std::min(n, *lo + step);
}

int build_s2_shared(Builder& B, std::vector<EdgeCtx>& xs, int Pr, int Pc, northup_stats* st) {
  const int G = static_cast<int>(xs.size());
  for (EdgeCtx& x : xs) {
    x.a_share = Pc;
    x.b_share = Pr;
    x.bfirst = -1;   // the shared plan is emitted in lock step by the drain-tail builder
  }
  S2Shape s{};
  int rc = choose_s2(xs[0], &s);
  if (rc) return rc;
  for (const EdgeCtx& x : xs)
    if (x.cap && s.bytes > x.cap)
      return fail(NU_ENOMEM, "HBM node %d capacity %llu B below the shared S2 block", x.hbm_node,
                  (unsigned long long)x.cap);
  const EdgeCtx& x0 = xs[0];
  const int64_t m = x0.r1 - x0.r0, n = x0.c1 - x0.c0, K = x0.K;
  const int64_t lda = x0.lda, ldb = x0.ldb, ldc = x0.ldc;
  std::vector<S2Layout> L(G);
  for (int w = 0; w < G; ++w) L[w] = layout_s2(B, s, xs[w].hbm_node, w, K);
  const S2Layout& Y = L[0];   // offsets are the same in every worker's arena
  s2_stats(s, st);
  st->shared_staging = 1;
  const int64_t kmain = K - s.tail;

  // One shared slot region (rows x cols at offset `off`, leading dim `ld`):
  // A side pieces split rows among the Pc row peers, B side pieces split
  // columns among the Pr column peers.
  struct Side {
    bool a;
    int hb;                      // user buffer (root tier)
    int64_t hld;                 // its leading dimension
    std::vector<int64_t> src;    // per worker: root offset of the region's origin
    int64_t off, ld, rows, cols;
  };
  auto idx = [&](const Side& sd, int w) { return sd.a ? w % Pc : w / Pc; };
  auto peer = [&](const Side& sd, int w, int q) { return sd.a ? (w / Pc) * Pc + q : q * Pc + w % Pc; };
  auto sub = [&](const Side& sd, int q, int64_t* r0, int64_t* nr, int64_t* c0, int64_t* nc) {
    int64_t lo, hi;
    piece_range(sd.a ? sd.rows : sd.cols, sd.a ? Pc : Pr, q, &lo, &hi);
    *r0 = sd.a ? lo : 0;
    *nr = sd.a ? hi - lo : sd.rows;
    *c0 = sd.a ? 0 : lo;
    *nc = sd.a ? sd.cols : hi - lo;
  };
  auto load = [&](const Side& sd) {        // own piece over PCIe (data_down)
    for (int w = 0; w < G; ++w) {
      int64_t r0, nr, c0, nc;
      sub(sd, idx(sd, w), &r0, &nr, &c0, &nc);
      if (nr <= 0 || nc <= 0) continue;
      const int64_t so = sd.src[w] + r0 * sd.hld + c0, d = sd.off + r0 * sd.ld + c0;
      B.emit(make_copy(w, S_H2D, sd.hb, so, sd.hld, L[w].arena, d, sd.ld, nr, nc),
             {{sd.hb, so, sd.hld, nr, nc, false}, {L[w].arena, d, sd.ld, nr, nc, true}});
      st->bytes_h2d += 4ull * nr * nc;
    }
  };
  auto pull = [&](const Side& sd) {        // the peers' pieces over NVLink
    const int parts = sd.a ? Pc : Pr;
    for (int w = 0; w < G; ++w)
      for (int q = 0; q < parts; ++q) {
        if (q == idx(sd, w)) continue;
        int64_t r0, nr, c0, nc;
        sub(sd, q, &r0, &nr, &c0, &nc);
        if (nr <= 0 || nc <= 0) continue;
        const int src = L[peer(sd, w, q)].arena;
        const int64_t d = sd.off + r0 * sd.ld + c0;
        B.emit(make_copy(w, S_D2D, src, d, sd.ld, L[w].arena, d, sd.ld, nr, nc),
               {{src, d, sd.ld, nr, nc, false}, {L[w].arena, d, sd.ld, nr, nc, true}});
        st->bytes_p2p += 4ull * nr * nc;
      }
  };
  auto side = [&](bool a, int64_t off, int64_t ld, int64_t rows, int64_t cols, auto src_of) {
    Side sd{a, a ? x0.A : x0.Bb, a ? lda : ldb, std::vector<int64_t>(G), off, ld, rows, cols};
    for (int w = 0; w < G; ++w) sd.src[w] = src_of(xs[w]);
    return sd;
  };

  int panel_it = 0, strip_it = 0;
  for (int64_t i0 = 0; i0 < m; i0 += s.bm) {
    const int64_t bm = std::min(s.bm, m - i0);
    for (int64_t j0 = 0; j0 < n; j0 += s.bn) {
      const int64_t bn = std::min(s.bn, n - j0);
      const int64_t npan = kmain > 0 ? cdiv(kmain, s.bk) : 0;
      const int64_t ntail_pieces = s.tail > 0 ? cdiv(s.tail, s.bk) : 0;
      int64_t pieces_done = 0;
      auto load_tail_piece = [&](int64_t pc) {
        const int64_t k0 = kmain + pc * s.bk, kk = std::min(s.bk, K - k0);
        Side sb = side(false, Y.offBT + (k0 - kmain) * Y.ldBs, Y.ldBs, kk, bn,
                       [&](const EdgeCtx& x) { return k0 * ldb + x.ac0 + j0; });
        load(sb);
        pull(sb);
        for (int w = 0; w < G; ++w) emit_tail_split(B, w, L[w], s, bn, k0 - kmain, kk);
      };
      for (int64_t p = 0; p < npan; ++p, ++panel_it) {
        const int sl = panel_it % kSlots;
        const int64_t k0 = p * s.bk, kk = std::min(s.bk, kmain - k0);
        Side sa = side(true, Y.offSA[sl], Y.ldA, bm, kk,
                       [&](const EdgeCtx& x) { return (x.ar0 + i0) * lda + k0; });
        Side sb = side(false, Y.offSB[sl], Y.ldBs, kk, bn,
                       [&](const EdgeCtx& x) { return k0 * ldb + x.ac0 + j0; });
        load(sa);
        load(sb);
        pull(sa);
        pull(sb);
        // the leaf ops of build_s2 (first panel as a 4 x 4 sub-block grid)
        const int64_t gb = (p == 0 && bm >= 4096 && bn >= 4096) ? 4 : 1;
        const int64_t sbm = rup(cdiv(bm, gb), 256), sbn = rup(cdiv(bn, gb), 256);
        for (int w = 0; w < G; ++w) {
          const int ar = L[w].arena;
          for (int64_t jj = 0; jj < bn; jj += sbn) {
            const int64_t cn = std::min(sbn, bn - jj);
            for (int64_t ii = 0; ii < bm; ii += sbm) {
              const int64_t rm = std::min(sbm, bm - ii);
              const int64_t ao = Y.offSA[sl] + ii * Y.ldA, bo = Y.offSB[sl] + jj,
                            co = Y.offC + ii * Y.ldC + jj;
              B.emit(make_leaf(w, ar, ao, Y.ldA, ar, bo, Y.ldBs, ar, co, Y.ldC, rm, cn, kk, p > 0 ? 1 : 0),
                     {{ar, ao, Y.ldA, rm, kk, false}, {ar, bo, Y.ldBs, kk, cn, false},
                      {ar, co, Y.ldC, rm, cn, true}});
              st->leaf_launches++;
            }
          }
        }
        const int64_t skip = std::min<int64_t>(2, std::max<int64_t>(0, npan - 1));
        while (pieces_done < ntail_pieces && p >= skip &&
               (pieces_done + 1) * (npan - skip) <= (p + 1 - skip) * ntail_pieces)
          load_tail_piece(pieces_done++);
      }
      while (pieces_done < ntail_pieces) load_tail_piece(pieces_done++);
      if (s.tail > 0) {
        for (int64_t r = 0, rr = 0; r < bm; r += rr, ++strip_it) {
          rr = next_strip(bm, r, s.sr);
          const int sl = strip_it % kSlots;
          Side sa = side(true, Y.offAT[sl], Y.ldAt, rr, s.tail,
                         [&](const EdgeCtx& x) { return (x.ar0 + i0 + r) * lda + kmain; });
          load(sa);
          pull(sa);
          for (int w = 0; w < G; ++w) {
            const int ar = L[w].arena;
            const int64_t co = Y.offC + r * Y.ldC;
            emit_tail_leaf(B, w, L[w], s, ar, Y.offAT[sl], Y.ldAt, co, Y.ldC, rr, bn, kmain > 0 ? 1 : 0);
            st->leaf_launches++;
            const int64_t dst = (xs[w].ar0 + i0 + r) * ldc + xs[w].ac0 + j0;
            B.emit(make_copy(w, S_D2H, ar, co, Y.ldC, x0.C, dst, ldc, rr, bn),
                   {{ar, co, Y.ldC, rr, bn, false}, {x0.C, dst, ldc, rr, bn, true}});
            st->bytes_d2h += 4ull * rr * bn;
          }
        }
      } else {
        for (int w = 0; w < G; ++w) {
          const int64_t dst = (xs[w].ar0 + i0) * ldc + xs[w].ac0 + j0;
          B.emit(make_copy(w, S_D2H, L[w].arena, Y.offC, Y.ldC, x0.C, dst, ldc, bm, bn),
                 {{L[w].arena, Y.offC, Y.ldC, bm, bn, false}, {x0.C, dst, ldc, bm, bn, true}});
          st->bytes_d2h += 4ull * bm * bn;
        }
      }
    }
  }
  return B.overflow ? fail(NU_ENOTSUP, "dependency fan-in above 16") : 0;
}

// ---------------------------------------------------------------- S1
int build_s1(const EdgeCtx& x, northup_stats* st) {
  Builder& B = *x.B;
  const int w = x.worker;
  const int64_t m = x.r1 - x.r0, n = x.c1 - x.c0, K = x.K;
  const uint64_t cap = x.cap ? x.cap : (uint64_t(1) << 62);
  int64_t bm = x.obm > 0 ? std::min(x.obm, m) : std::min<int64_t>(m, 4096);
  int64_t bn = x.obn > 0 ? std::min(x.obn, n) : std::min<int64_t>(n, 4096);
  int64_t bk = x.obk > 0 ? std::min(x.obk, rup(K, 4)) : std::min<int64_t>(rup(K, 4), x.kc);
  auto bytes_of = [&](int64_t bm_, int64_t bn_, int64_t bk_) -> uint64_t {
    return 4ull * (2ull * bm_ * pad_ld(K)             // two row shards (next prefetches)
                   + 2ull * bm_ * pad_ld(bn_)         // double-buffered C block
                   + uint64_t(kSlots) * bk_ * pad_ld(bn_)) +
           leaf_scratch(bm_, bn_, x.kc);
  };
  while (bytes_of(bm, bn, bk) > cap) {
    if (bm > 128 && x.obm <= 0) bm = rup(cdiv(bm, 2), 128);
    else if (bn > 256 && x.obn <= 0) bn = rup(cdiv(bn, 2), 256);
    else return fail(NU_ENOMEM, "HBM node %d capacity too small for S1 blocks", x.hbm_node);
  }
  const uint64_t bytes = bytes_of(bm, bn, bk);
  const int arena = B.add_buf(B_ARENA, x.hbm_node, w, bytes);
  set_scratch(B.P, w, arena, bytes, leaf_scratch(bm, bn, x.kc));
  const int64_t ldAs = pad_ld(K), ldC = pad_ld(bn), ldB = pad_ld(bn);
  int64_t off = 0, offAs[2], offC[2], offB[kSlots];
  for (int i = 0; i < 2; ++i) { offAs[i] = off; off += bm * ldAs; }
  for (int i = 0; i < 2; ++i) { offC[i] = off; off += bm * ldC; }
  for (int i = 0; i < kSlots; ++i) { offB[i] = off; off += bk * ldB; }
  if (w == 0) {
    st->bm = bm;
    st->bn = bn;
    st->bk = bk;
    st->hbm_peak_bytes = bytes;
    st->schedule = NU_SCHED_S1;
  }
  int shard = 0, cblk = 0, pit = 0;
  for (int64_t i0 = 0; i0 < m; i0 += bm, ++shard) {
    const int64_t rm = std::min(bm, m - i0);
    const int64_t gr = x.ar0 + i0;
    const int as = shard & 1;
    // row shard m moves to level l+1 once and stays
    B.emit(make_copy(w, S_H2D, x.A, gr * x.lda, x.lda, arena, offAs[as], ldAs, rm, K),
           {{x.A, gr * x.lda, x.lda, rm, K, false}, {arena, offAs[as], ldAs, rm, K, true}});
    st->bytes_h2d += static_cast<uint64_t>(rm) * K * 4;
    for (int64_t j0 = 0; j0 < n; j0 += bn, ++cblk) {
      const int64_t cn = std::min(bn, n - j0);
      const int64_t gc = x.ac0 + j0;
      const int cb = cblk & 1;
      for (int64_t k0 = 0; k0 < K; k0 += bk, ++pit) {
        const int64_t kk = std::min(bk, K - k0);
        const int sl = pit % kSlots;
        B.emit(make_copy(w, S_H2D, x.Bb, k0 * x.ldb + gc, x.ldb, arena, offB[sl], ldB, kk, cn),
               {{x.Bb, k0 * x.ldb + gc, x.ldb, kk, cn, false}, {arena, offB[sl], ldB, kk, cn, true}});
        st->bytes_h2d += static_cast<uint64_t>(kk) * cn * 4;
        B.emit(make_leaf(w, arena, offAs[as] + k0, ldAs, arena, offB[sl], ldB, arena, offC[cb], ldC,
                         rm, cn, kk, k0 > 0 ? 1 : 0),
               {{arena, offAs[as] + k0, ldAs, rm, kk, false},
                {arena, offB[sl], ldB, kk, cn, false},
                {arena, offC[cb], ldC, rm, cn, true}});
        st->leaf_launches++;
      }
      B.emit(make_copy(w, S_D2H, arena, offC[cb], ldC, x.C, gr * x.ldc + gc, x.ldc, rm, cn),
             {{arena, offC[cb], ldC, rm, cn, false}, {x.C, gr * x.ldc + gc, x.ldc, rm, cn, true}});
      st->bytes_d2h += static_cast<uint64_t>(rm) * cn * 4;
    }
  }
  return 0;
}

// In-HBM (single-node HBM tree, CS4): the leaf runs directly on the caller's
// device buffers; operands whose layout TMA cannot address are first copied
// into padded arena buffers (R16 layout transformation during move_data).
int build_in_hbm(Builder& B, int node, int64_t M, int64_t N, int64_t K, int A, int Bb, int C,
                 bool a_ok, bool b_ok, northup_stats* st) {
  const int64_t ldA = pad_ld(K), ldB = pad_ld(N);
  uint64_t bytes = 0;
  if (!a_ok) bytes += 4ull * M * ldA;
  if (!b_ok) bytes += 4ull * K * ldB;
  const uint64_t scr = leaf_scratch(M, N, B.P->kc);
  bytes += scr;
  int64_t offA = 0, offB = a_ok ? 0 : M * ldA;
  const int arena = B.add_buf(B_ARENA, node, 0, bytes);
  set_scratch(B.P, 0, arena, bytes, scr);
  int a = A, b = Bb;
  int64_t la = K, lb = N, oa = 0, ob = 0;
  if (!a_ok) {
    B.emit(make_copy(0, S_COMP, A, 0, K, arena, offA, ldA, M, K),
           {{A, 0, K, M, K, false}, {arena, offA, ldA, M, K, true}});
    st->bytes_d2d += 4ull * M * K;
    a = arena, la = ldA, oa = offA;
  }
  if (!b_ok) {
    B.emit(make_copy(0, S_COMP, Bb, 0, N, arena, offB, ldB, K, N),
           {{Bb, 0, N, K, N, false}, {arena, offB, ldB, K, N, true}});
    st->bytes_d2d += 4ull * K * N;
    b = arena, lb = ldB, ob = offB;
  }
  B.emit(make_leaf(0, a, oa, la, b, ob, lb, C, 0, N, M, N, K, 0),
         {{a, oa, la, M, K, false}, {b, ob, lb, K, N, false}, {C, 0, N, M, N, true}});
  st->leaf_launches++;
  st->bm = M;
  st->bn = N;
  st->bk = K;
  st->hbm_peak_bytes = bytes;
  st->schedule = NU_SCHED_AUTO;
  return 0;
}


// FILE root (S§8(a) a3): FILE -> HOST staging -> G x HBM -> SMEM/TMEM.
// K panels of A and B are read from the files into a ring of DRAM staging
// slots shared by all siblings (each file byte is read once per C-block round),
// every sibling copies its rows / columns of the panel to its HBM slots and
// accumulates into its resident C block; finished C blocks drain HBM -> DRAM
// strip by strip and are written back to the C file (Listing 4 file_write).
northup_op make_io(int io_worker, int op, int src, int64_t src_off, int64_t src_ld, int dst,
                   int64_t dst_off, int64_t dst_ld, int64_t rows, int64_t cols) {
  northup_op o = make_copy(io_worker, op == NU_OP_IO_WRITE ? S_IOW : S_IO, src, src_off, src_ld, dst, dst_off,
                           dst_ld, rows, cols);
  o.op = op;
  return o;
}

int build_file_root(Builder& B, const northup_tree_s* t, int staging, const std::vector<int>& hbm,
                    int64_t M, int64_t N, int64_t K, int A, int Bb, int C, int64_t kc,
                    int64_t a_panel_k, northup_stats* st) {
  const int G = static_cast<int>(hbm.size());
  const int io = G;   // the I/O pseudo-worker
  // a K shorter than the panel is one panel of width K (the file layout agrees: R15)
  const int64_t bk = std::min<int64_t>(a_panel_k > 0 ? a_panel_k : kc, std::max<int64_t>(K, 1));
  // per-worker regions and one common C-block shape that fits every HBM node
  std::vector<int64_t> r0(G), r1(G), c0(G), c1(G);
  int64_t mmax = 0, nmax = 0;
  uint64_t cap = uint64_t(1) << 62;
  for (int w = 0; w < G; ++w) {
    int rc = region_of(G, M, N, w, &r0[w], &r1[w], &c0[w], &c1[w]);
    if (rc) return rc;
    mmax = std::max(mmax, r1[w] - r0[w]);
    nmax = std::max(nmax, c1[w] - c0[w]);
    if (t->nodes[hbm[w]].capacity) cap = std::min<uint64_t>(cap, t->nodes[hbm[w]].capacity);
  }
  auto hbm_bytes = [&](int64_t bm, int64_t bn) {
    return 4ull * (uint64_t(bm) * pad_ld(bn) +
                   uint64_t(kSlots) * (uint64_t(bm) * pad_ld(bk) + uint64_t(bk) * pad_ld(bn))) +
           leaf_scratch(bm, bn, kc);
  };
  int64_t bm = mmax, bn = nmax;
  while (hbm_bytes(bm, bn) > cap) {
    if (bm > 128) bm = rup(cdiv(bm, 2), 128);
    else if (bn > 256) bn = rup(cdiv(bn, 2), 256);
    else return fail(NU_ENOMEM, "HBM capacity %llu B below the minimum block", (unsigned long long)cap);
  }
  const int64_t nbr = cdiv(mmax, bm), nbc = cdiv(nmax, bn), rounds = nbr * nbc;
  const int64_t sr = std::min<int64_t>(bm, rup(cdiv(bm, 8), 128));   // drain strip rows
  // DRAM staging: R panel slots (A panel M x bk, B panel bk x N) + 2 C strips per GPU
  const uint64_t dcap = t->nodes[staging].capacity ? t->nodes[staging].capacity : uint64_t(1) << 62;
  const uint64_t panel_e = uint64_t(M) * bk + uint64_t(bk) * N;
  const uint64_t cstage_e = uint64_t(G) * 2 * sr * bn;
  int R = kSlots;
  while (R > 1 && 4ull * (R * panel_e + cstage_e) > dcap) --R;
  if (4ull * (R * panel_e + cstage_e) > dcap)
    return fail(NU_ENOMEM, "staging node %d capacity %llu B below one panel + C strips", staging,
                (unsigned long long)dcap);
  const int dram = B.add_buf(B_DRAM, staging, -1, 4ull * (R * panel_e + cstage_e));
  std::vector<int> arena(G);
  for (int w = 0; w < G; ++w) {
    arena[w] = B.add_buf(B_ARENA, hbm[w], w, hbm_bytes(bm, bn));
    set_scratch(B.P, w, arena[w], hbm_bytes(bm, bn), leaf_scratch(bm, bn, kc));
  }
  const int64_t ldC = pad_ld(bn), ldA = pad_ld(bk), ldB = pad_ld(bn);
  const int64_t offC = 0;
  int64_t offSA[kSlots], offSB[kSlots];
  for (int i = 0, off = 0; i < kSlots; ++i) {
    offSA[i] = offC + bm * ldC + i * (bm * ldA + bk * ldB);
    offSB[i] = offSA[i] + bm * ldA;
    (void)off;
  }
  auto slotA = [&](int s) { return int64_t(s) * int64_t(panel_e); };
  auto slotB = [&](int s) { return int64_t(s) * int64_t(panel_e) + M * bk; };
  auto cst = [&](int w, int j) { return int64_t(R) * int64_t(panel_e) + (int64_t(w) * 2 + j) * sr * bn; };
  st->bm = bm;
  st->bn = bn;
  st->bk = bk;
  st->hbm_peak_bytes = hbm_bytes(bm, bn);
  st->schedule = NU_SCHED_S2;
  const int64_t npan = cdiv(K, bk);
  int64_t gp = 0;               // global panel counter (DRAM ring)
  std::vector<int64_t> hslot(G, 0), cstrip(G, 0);
  for (int64_t r = 0; r < rounds; ++r) {
    const int64_t bi = r / nbc, bj = r % nbc;
    for (int64_t p = 0; p < npan; ++p, ++gp) {
      const int s = static_cast<int>(gp % R);
      const int64_t k0 = p * bk, kk = std::min(bk, K - k0);
      // file -> DRAM: one sequential read per panel when A is K-panel-major
      if (a_panel_k > 0)
        B.emit(make_io(io, NU_OP_IO_READ, A, k0 * M, kk, dram, slotA(s), kk, M, kk),
               {{A, k0 * M, kk, M, kk, false}, {dram, slotA(s), kk, M, kk, true}});
      else
        B.emit(make_io(io, NU_OP_IO_READ, A, k0, K, dram, slotA(s), kk, M, kk),
               {{A, k0, K, M, kk, false}, {dram, slotA(s), kk, M, kk, true}});
      B.emit(make_io(io, NU_OP_IO_READ, Bb, k0 * N, N, dram, slotB(s), N, kk, N),
             {{Bb, k0 * N, N, kk, N, false}, {dram, slotB(s), N, kk, N, true}});
      st->bytes_file_read += 4ull * (uint64_t(M) * kk + uint64_t(kk) * N);
      for (int w = 0; w < G; ++w) {
        const int64_t i0 = bi * bm, j0 = bj * bn;
        const int64_t m = std::min(bm, (r1[w] - r0[w]) - i0), n = std::min(bn, (c1[w] - c0[w]) - j0);
        if (m <= 0 || n <= 0) continue;
        const int64_t gr = r0[w] + i0, gc = c0[w] + j0;
        const int sl = static_cast<int>(hslot[w]++ % kSlots);
        B.emit(make_copy(w, S_H2D, dram, slotA(s) + gr * kk, kk, arena[w], offSA[sl], ldA, m, kk),
               {{dram, slotA(s) + gr * kk, kk, m, kk, false}, {arena[w], offSA[sl], ldA, m, kk, true}});
        B.emit(make_copy(w, S_H2D, dram, slotB(s) + gc, N, arena[w], offSB[sl], ldB, kk, n),
               {{dram, slotB(s) + gc, N, kk, n, false}, {arena[w], offSB[sl], ldB, kk, n, true}});
        st->bytes_h2d += 4ull * (uint64_t(m) * kk + uint64_t(kk) * n);
        B.emit(make_leaf(w, arena[w], offSA[sl], ldA, arena[w], offSB[sl], ldB, arena[w], offC, ldC,
                         m, n, kk, p > 0 ? 1 : 0),
               {{arena[w], offSA[sl], ldA, m, kk, false},
                {arena[w], offSB[sl], ldB, kk, n, false},
                {arena[w], offC, ldC, m, n, true}});
        st->leaf_launches++;
      }
    }
    // drain: HBM -> DRAM strips -> C file (Listing 4: file_write)
    for (int w = 0; w < G; ++w) {
      const int64_t i0 = bi * bm, j0 = bj * bn;
      const int64_t m = std::min(bm, (r1[w] - r0[w]) - i0), n = std::min(bn, (c1[w] - c0[w]) - j0);
      if (m <= 0 || n <= 0) continue;
      const int64_t gr = r0[w] + i0, gc = c0[w] + j0;
      for (int64_t q = 0; q < m; q += sr) {
        const int64_t rr = std::min(sr, m - q);
        const int j = static_cast<int>(cstrip[w]++ % 2);
        B.emit(make_copy(w, S_D2H, arena[w], offC + q * ldC, ldC, dram, cst(w, j), n, rr, n),
               {{arena[w], offC + q * ldC, ldC, rr, n, false}, {dram, cst(w, j), n, rr, n, true}});
        st->bytes_d2h += 4ull * rr * n;
        B.emit(make_io(io, NU_OP_IO_WRITE, dram, cst(w, j), n, C, (gr + q) * N + gc, N, rr, n),
               {{dram, cst(w, j), n, rr, n, false}, {C, (gr + q) * N + gc, N, rr, n, true}});
        st->bytes_file_write += 4ull * rr * n;
      }
    }
  }
  return B.overflow ? fail(NU_ENOTSUP, "dependency fan-in above 16") : 0;
}

// FILE root -> HBM siblings directly (S§8(f) NEXT-4: the GDS edge, P:240's
// mmap alternative / GPUfs P:45): no DRAM staging level.  Each sibling keeps
// its C block resident in HBM and reads the K panels of A (K-panel-major file,
// R15) and B (row-major) from the files straight into its HBM panel slots;
// finished C blocks are written from HBM to the C file.  The I/O thread does
// the transfers with cuFile (GPUDirect Storage; compat mode where the file
// system has no GDS support) and falls back to a pinned bounce buffer when
// cuFile cannot be opened.  Slots have unpadded rows where the file's rows are
// contiguous, so one panel is one read.
int build_file_direct(Builder& B, const northup_tree_s* t, const std::vector<int>& hbm, int64_t M,
                      int64_t N, int64_t K, int A, int Bb, int C, int64_t kc, int64_t a_panel_k,
                      northup_stats* st) {
  const int G = static_cast<int>(hbm.size());
  const int io = G;   // the I/O pseudo-worker
  const int64_t bk = std::min<int64_t>(a_panel_k > 0 ? a_panel_k : kc, std::max<int64_t>(K, 1));
  std::vector<int64_t> r0(G), r1(G), c0(G), c1(G);
  int64_t mmax = 0, nmax = 0;
  uint64_t cap = uint64_t(1) << 62;
  for (int w = 0; w < G; ++w) {
    int rc = region_of(G, M, N, w, &r0[w], &r1[w], &c0[w], &c1[w]);
    if (rc) return rc;
    mmax = std::max(mmax, r1[w] - r0[w]);
    nmax = std::max(nmax, c1[w] - c0[w]);
    if (t->nodes[hbm[w]].capacity) cap = std::min<uint64_t>(cap, t->nodes[hbm[w]].capacity);
  }
  // A slot rows: bk when the panel width keeps 16-B rows (TMA), else padded
  const bool bk4 = bk % 4 == 0 && K % 4 == 0;
  auto lda_of = [&](int64_t kk) { return bk4 ? kk : pad_ld(kk); };
  auto hbm_bytes = [&](int64_t bm, int64_t bn) {
    const int64_t ldb = (bn == N && N % 4 == 0) ? bn : pad_ld(bn);
    return 4ull * (uint64_t(bm) * pad_ld(bn) + uint64_t(kSlots) * (uint64_t(bm) * lda_of(bk) + uint64_t(bk) * ldb)) +
           leaf_scratch(bm, bn, kc);
  };
  int64_t bm = mmax, bn = nmax;
  while (hbm_bytes(bm, bn) > cap) {
    if (bm > 128) bm = rup(cdiv(bm, 2), 128);
    else if (bn > 256) bn = rup(cdiv(bn, 2), 256);
    else return fail(NU_ENOMEM, "HBM capacity %llu B below the minimum block", (unsigned long long)cap);
  }
  const int64_t ldC = pad_ld(bn), ldBs = (bn == N && N % 4 == 0) ? bn : pad_ld(bn);
  std::vector<int> arena(G);
  for (int w = 0; w < G; ++w) {
    arena[w] = B.add_buf(B_ARENA, hbm[w], w, hbm_bytes(bm, bn));
    set_scratch(B.P, w, arena[w], hbm_bytes(bm, bn), leaf_scratch(bm, bn, kc));
  }
  st->bm = bm;
  st->bn = bn;
  st->bk = bk;
  st->hbm_peak_bytes = hbm_bytes(bm, bn);
  st->schedule = NU_SCHED_S2;
  const int64_t npan = cdiv(K, bk);
  std::vector<int64_t> slot(G, 0);
  const int64_t nbr = cdiv(mmax, bm), nbc = cdiv(nmax, bn);
  for (int64_t bi = 0; bi < nbr; ++bi)
    for (int64_t bj = 0; bj < nbc; ++bj) {
      for (int64_t p = 0; p < npan; ++p) {
        const int64_t k0 = p * bk, kk = std::min(bk, K - k0);
        const int64_t ldA = lda_of(kk);
        for (int w = 0; w < G; ++w) {
          const int64_t i0 = bi * bm, j0 = bj * bn;
          const int64_t m = std::min(bm, (r1[w] - r0[w]) - i0), n = std::min(bn, (c1[w] - c0[w]) - j0);
          if (m <= 0 || n <= 0) continue;
          const int64_t gr = r0[w] + i0, gc = c0[w] + j0;
          const int sl = static_cast<int>(slot[w]++ % kSlots);
          const int64_t offSA = bm * ldC + sl * (bm * lda_of(bk) + bk * ldBs);
          const int64_t offSB = offSA + bm * lda_of(bk);
          // file -> HBM: A rows of this block in panel p, B rows of panel p
          if (a_panel_k > 0)
            B.emit(make_io(io, NU_OP_IO_READ, A, k0 * M + gr * kk, kk, arena[w], offSA, ldA, m, kk),
                   {{A, k0 * M + gr * kk, kk, m, kk, false}, {arena[w], offSA, ldA, m, kk, true}});
          else
            B.emit(make_io(io, NU_OP_IO_READ, A, gr * K + k0, K, arena[w], offSA, ldA, m, kk),
                   {{A, gr * K + k0, K, m, kk, false}, {arena[w], offSA, ldA, m, kk, true}});
          B.emit(make_io(io, NU_OP_IO_READ, Bb, k0 * N + gc, N, arena[w], offSB, ldBs, kk, n),
                 {{Bb, k0 * N + gc, N, kk, n, false}, {arena[w], offSB, ldBs, kk, n, true}});
          st->bytes_file_read += 4ull * (uint64_t(m) * kk + uint64_t(kk) * n);
          B.emit(make_leaf(w, arena[w], offSA, ldA, arena[w], offSB, ldBs, arena[w], 0, ldC, m, n, kk,
                           p > 0 ? 1 : 0),
                 {{arena[w], offSA, ldA, m, kk, false}, {arena[w], offSB, ldBs, kk, n, false},
                  {arena[w], 0, ldC, m, n, true}});
          st->leaf_launches++;
        }
      }
      // HBM -> file: the C block (Listing 4 file_write from the HBM level)
      for (int w = 0; w < G; ++w) {
        const int64_t i0 = bi * bm, j0 = bj * bn;
        const int64_t m = std::min(bm, (r1[w] - r0[w]) - i0), n = std::min(bn, (c1[w] - c0[w]) - j0);
        if (m <= 0 || n <= 0) continue;
        const int64_t gr = r0[w] + i0, gc = c0[w] + j0;
        B.emit(make_io(io, NU_OP_IO_WRITE, arena[w], 0, ldC, C, gr * N + gc, N, m, n),
               {{arena[w], 0, ldC, m, n, false}, {C, gr * N + gc, N, m, n, true}});
        st->bytes_file_write += 4ull * m * n;
      }
    }
  return B.overflow ? fail(NU_ENOTSUP, "dependency fan-in above 16") : 0;
}

}  // namespace

// ------------------------------------------------- NU_SCHED_QUEUE (NEXT-2)
// The paper's runtime keeps a task queue at each node and
// balances work by popping local tasks and stealing remote ones (P:393-395,
// there between CPU and GPU).  Here the tasks are C tiles of an M x N GEMM and
// the queues belong to the HBM siblings: two tiles per sibling, each an
// S2 sub-problem with its C tile resident in one of two tile buffers (so the
// next tile's panels stream while the previous one drains).
int choose_queue(const northup_tree_s* t, const std::vector<int>& hbm, int64_t M, int64_t N, int64_t K,
                 int64_t kc, int tiles, QueueShape* q) {
  const int G = static_cast<int>(hbm.size());
  uint64_t cap = 0;
  for (int h : hbm)
    if (t->nodes[h].capacity) cap = cap ? std::min(cap, t->nodes[h].capacity) : t->nodes[h].capacity;
  int Pr = 1, Pc = 1;
  partition_grid(G, M, N, &Pr, &Pc);
  const int64_t bk = std::min<int64_t>(std::max<int64_t>(kc, 4), rup(K, 4));
  auto bytes = [&](int64_t tm, int64_t tn) {
    return 4ull * (2ull * tm * pad_ld(tn) + uint64_t(kSlots) * (uint64_t(tm) * pad_ld(bk) + uint64_t(bk) * pad_ld(tn))) +
           leaf_scratch(tm, tn, kc);
  };
  // `tiles` (default 2) tiles per sibling: split each sibling's region, one
  // factor of 2 at a time, in the direction that adds fewer PCIe bytes (every
  // tile streams its A rows and B columns once: H2D = 4K (M Tc + N Tr));
  // refine further only until it fits
  int64_t Tr = Pr, Tc = Pc;
  for (int f = 1; f < std::max(tiles, 2); f *= 2) {
    if (M * Tc + N * 2 * Tr <= M * 2 * Tc + N * Tr) Tr = std::min<int64_t>(M, 2 * Tr);
    else Tc = std::min<int64_t>(N, 2 * Tc);
  }
  for (;;) {
    const int64_t tm = rup(cdiv(M, Tr), 8), tn = rup(cdiv(N, Tc), 8);
    if (!cap || bytes(tm, tn) <= cap) {
      q->tm = tm;
      q->tn = tn;
      q->bk = bk;
      q->Tr = cdiv(M, tm);
      q->Tc = cdiv(N, tn);
      q->arena_bytes = bytes(tm, tn);
      q->scratch_bytes = leaf_scratch(tm, tn, kc);
      return 0;
    }
    if (tm <= 8 && tn <= 8)
      return fail(NU_ENOMEM, "HBM capacity %llu B below the smallest queue tile", (unsigned long long)cap);
    if (tm >= tn && tm > 8) Tr = std::min<int64_t>(M, Tr * 2);
    else Tc = std::min<int64_t>(N, Tc * 2);
  }
}

std::vector<std::vector<int64_t>> queue_initial(int G, const QueueShape& q) {
  const int64_t T = q.Tr * q.Tc;
  std::vector<std::vector<int64_t>> out(G);
  for (int w = 0; w < G; ++w)
    for (int64_t i = T * w / G; i < T * (w + 1) / G; ++i) out[w].push_back(i);
  return out;
}

void emit_task(Builder& B, int w, int arena, const QueueShape& q, int64_t task, int cslot, int64_t* pctr,
               int A, int Bb, int C, int64_t M, int64_t N, int64_t K, northup_stats* st) {
  const int64_t ti = task / q.Tc, tj = task % q.Tc;
  const int64_t i0 = ti * q.tm, j0 = tj * q.tn;
  const int64_t m = std::min(q.tm, M - i0), n = std::min(q.tn, N - j0);
  const int64_t ldC = pad_ld(q.tn), ldA = pad_ld(q.bk), ldB = pad_ld(q.tn);
  const int64_t offC = static_cast<int64_t>(cslot) * q.tm * ldC;
  const int64_t base = 2 * q.tm * ldC;
  for (int64_t k0 = 0, p = 0; k0 < K; k0 += q.bk, ++p) {
    const int64_t kk = std::min(q.bk, K - k0);
    const int sl = static_cast<int>((*pctr)++ % kSlots);
    const int64_t offA = base + sl * (q.tm * ldA + q.bk * ldB), offB = offA + q.tm * ldA;
    B.emit(make_copy(w, S_H2D, A, i0 * K + k0, K, arena, offA, ldA, m, kk),
           {{A, i0 * K + k0, K, m, kk, false}, {arena, offA, ldA, m, kk, true}});
    B.emit(make_copy(w, S_H2D, Bb, k0 * N + j0, N, arena, offB, ldB, kk, n),
           {{Bb, k0 * N + j0, N, kk, n, false}, {arena, offB, ldB, kk, n, true}});
    st->bytes_h2d += 4ull * (uint64_t(m) * kk + uint64_t(kk) * n);
    B.emit(make_leaf(w, arena, offA, ldA, arena, offB, ldB, arena, offC, ldC, m, n, kk, p > 0 ? 1 : 0),
           {{arena, offA, ldA, m, kk, false}, {arena, offB, ldB, kk, n, false}, {arena, offC, ldC, m, n, true}});
    st->leaf_launches++;
  }
  B.emit(make_copy(w, S_D2H, arena, offC, ldC, C, i0 * N + j0, N, m, n),
         {{arena, offC, ldC, m, n, false}, {C, i0 * N + j0, N, m, n, true}});
  st->bytes_d2h += 4ull * m * n;
}

// Which HBM nodes compute, and what sits above them.
int build_plan(const northup_tree_s* t, int64_t M, int64_t N, int64_t K, const northup_gemm_opts* o,
               Plan* out) {
  return build_plan_ex(t, M, N, K, o, true, true, out);
}

static int build_plan_impl(const northup_tree_s* t, int64_t M, int64_t N, int64_t K,
                           const northup_gemm_opts* o, bool a_aligned, bool b_aligned, Plan* out);

int build_plan_ex(const northup_tree_s* t, int64_t M, int64_t N, int64_t K,
                  const northup_gemm_opts* o, bool a_aligned, bool b_aligned, Plan* out) {
  int rc = build_plan_impl(t, M, N, K, o, a_aligned, b_aligned, out);
  if (rc) return rc;
  // leaf_launches counts kernel launches: the leaf issues one launch per
  // k_chunk panel of each LEAF op (leaf_host.cu, kPanelChunks).
  int64_t n = 0;
  for (const northup_op& op : out->ops)
    if (op.op == NU_OP_LEAF) n += kPanelChunks > 0 ? cdiv(op.k, kPanelChunks * out->kc) : 1;
  out->stats.leaf_launches = n;
  return 0;
}

static int build_plan_impl(const northup_tree_s* t, int64_t M, int64_t N, int64_t K,
                           const northup_gemm_opts* o, bool a_aligned, bool b_aligned, Plan* out) {
  int rc = validate_tree(t);
  if (rc) return rc;
  if (M < 0 || N < 0 || K < 0) return fail(NU_EINVAL, "negative dimension");
  Plan& P = *out;
  P = Plan();
  P.M = M;
  P.N = N;
  P.K = K;
  P.kc = (o && o->k_chunk > 0) ? o->k_chunk : kDefaultKChunk;
  if (P.kc % 4) return fail(NU_EINVAL, "k_chunk must be a multiple of 4");
  P.npass = o ? o->npass : 0;   // 0 = library default (leaf_host.cu)
  const int sched = o ? o->schedule : NU_SCHED_AUTO;
  if (sched < NU_SCHED_AUTO || sched > NU_SCHED_S2B) return fail(NU_EINVAL, "unknown schedule");
  Builder B;
  B.P = &P;
  const int A = B.add_buf(B_USER_A, 0, -1, 4ull * M * K);
  const int Bb = B.add_buf(B_USER_B, 0, -1, 4ull * K * N);
  const int C = B.add_buf(B_USER_C, 0, -1, 4ull * M * N);
  northup_stats& st = P.stats;
  st = northup_stats{};
  const nu::Node& root = t->nodes[0];

  if (root.storage == NU_HBM) {
    // single-node HBM tree (or HBM -> SMEM leaf): the in-HBM reference (CS4)
    P.root_is_device = true;
    P.num_workers = 1;
    P.worker_node.push_back(0);
    st.num_gpus = 1;
    if (M == 0 || N == 0 || K == 0) return 0;
    // Layout legality is decided by the executor against real pointers; the
    // plan assumes dense ld = K / N and records whether those are TMA-legal.
    rc = build_in_hbm(B, 0, M, N, K, A, Bb, C, a_aligned && K % 4 == 0, b_aligned && N % 4 == 0,
                      &st);
    st.ops = static_cast<int64_t>(P.ops.size());
    return rc;
  }
  if (root.storage == NU_FILE) {
    bool direct = !root.children.empty();
    for (int c : root.children) direct = direct && t->nodes[c].storage == NU_HBM;
    if (direct) {
      // FILE -> HBM siblings (the GDS edge, NEXT-4)
      std::vector<int> hbm(root.children.begin(), root.children.end());
      P.num_workers = static_cast<int>(hbm.size());
      P.worker_node = hbm;
      st.num_gpus = P.num_workers;
      P.file_root = true;
      if (M == 0 || N == 0 || K == 0) return 0;
      rc = build_file_direct(B, t, hbm, M, N, K, A, Bb, C, P.kc, o ? o->a_panel_k : 0, &st);
      st.ops = static_cast<int64_t>(P.ops.size());
      for (const northup_op& op : P.ops)
        if (op.op == NU_OP_IO_READ || op.op == NU_OP_IO_WRITE) st.copies++;
      return rc;
    }
    // FILE -> HOST (DRAM staging) -> HBM siblings
    if (root.children.size() != 1 || t->nodes[root.children[0]].storage != NU_HOST)
      return fail(NU_ENOTSUP, "a FILE root needs HBM children (GDS edge) or one HOST staging child");
    const int staging = root.children[0];
    std::vector<int> hbm;
    for (int c : t->nodes[staging].children) {
      if (t->nodes[c].storage != NU_HBM)
        return fail(NU_ENOTSUP, "staging node children must be HBM nodes (node %d is not)", c);
      hbm.push_back(c);
    }
    if (hbm.empty()) return fail(NU_EINVAL, "staging node has no HBM child");
    P.num_workers = static_cast<int>(hbm.size());
    P.worker_node = hbm;
    st.num_gpus = P.num_workers;
    P.file_root = true;
    if (M == 0 || N == 0 || K == 0) return 0;
    rc = build_file_root(B, t, staging, hbm, M, N, K, A, Bb, C, P.kc, o ? o->a_panel_k : 0, &st);
    st.ops = static_cast<int64_t>(P.ops.size());
    for (const northup_op& op : P.ops)
      if (op.op == NU_OP_COPY || op.op == NU_OP_IO_READ || op.op == NU_OP_IO_WRITE) st.copies++;
    return rc;
  }
  if (root.storage != NU_HOST) return fail(NU_EINVAL, "root must be FILE, HOST or HBM");

  // HOST root: its children must be the HBM siblings (branch parallelism).
  std::vector<int> hbm;
  for (int c : root.children) {
    if (t->nodes[c].storage != NU_HBM)
      return fail(NU_ENOTSUP, "HOST root children must be HBM nodes (node %d is not)", c);
    hbm.push_back(c);
  }
  if (hbm.empty()) return fail(NU_EINVAL, "HOST root has no HBM child");
  const int G = static_cast<int>(hbm.size());
  P.num_workers = G;
  P.worker_node = hbm;
  st.num_gpus = G;
  if (M == 0 || N == 0 || K == 0) return 0;
  if (sched == NU_SCHED_QUEUE) {
    // The executor pops tiles at run time; the plan API shows the schedule
    // with no steals: each sibling takes its own queue in order, siblings in
    // round-robin (every op, dependency and byte count is the same as at run
    // time; only the tile-to-sibling assignment is dynamic).
    if (t->local_node >= 0) return fail(NU_ENOTSUP, "NU_SCHED_QUEUE runs in one process");
    QueueShape q;
    rc = choose_queue(t, hbm, M, N, K, P.kc, o ? o->queue_tiles : 0, &q);
    if (rc) return rc;
    std::vector<int> arena(G);
    for (int w = 0; w < G; ++w) {
      arena[w] = B.add_buf(B_ARENA, hbm[w], w, q.arena_bytes);
      set_scratch(&P, w, arena[w], q.arena_bytes, q.scratch_bytes);
    }
    auto queues = queue_initial(G, q);
    std::vector<int64_t> pctr(G, 0), done(G, 0);
    for (bool more = true; more;) {
      more = false;
      for (int w = 0; w < G; ++w) {
        if (done[w] >= static_cast<int64_t>(queues[w].size())) continue;
        emit_task(B, w, arena[w], q, queues[w][done[w]], static_cast<int>(done[w] & 1), &pctr[w], A, Bb, C,
                  M, N, K, &st);
        ++done[w];
        more = true;
      }
    }
    st.bm = q.tm;
    st.bn = q.tn;
    st.bk = q.bk;
    st.tasks = q.Tr * q.Tc;
    st.hbm_peak_bytes = q.arena_bytes;
    st.schedule = NU_SCHED_QUEUE;
    st.ops = static_cast<int64_t>(P.ops.size());
    for (const northup_op& op : P.ops)
      if (op.op == NU_OP_COPY) st.copies++;
    return B.overflow ? fail(NU_ENOTSUP, "dependency fan-in above 16") : 0;
  }
  if (o && o->replicate_result && t->local_node < 0) {
    // replicate_result in one process: the plan pushes each drained C piece to
    // every sibling's replica (Builder::push_replicas)
    for (int w = 0; w < G; ++w) {
      const Node& n = t->nodes[hbm[w]];
      if (!n.replica || n.replica_bytes < 4ull * M * N)
        return fail(NU_EINVAL, "replicate_result: HBM node %d has no M x N replica buffer "
                               "(northup_tree_set_replica)", n.id);
    }
    for (int w = 0; w < G; ++w) B.replica.push_back(B.add_buf(B_REPLICA, hbm[w], w, 4ull * M * N));
    P.replica_push = true;
  }
  std::vector<EdgeCtx> xs;
  std::vector<int> uses;
  for (int w = 0; w < G; ++w) {
    EdgeCtx x{};
    x.B = &B;
    x.worker = w;
    x.hbm_node = hbm[w];
    x.A = A;
    x.Bb = Bb;
    x.C = C;
    x.lda = K;
    x.ldb = N;
    x.ldc = N;
    rc = region_of(G, M, N, w, &x.r0, &x.r1, &x.c0, &x.c1);
    if (rc) return rc;
    x.ar0 = x.r0;
    x.ac0 = x.c0;
    if (t->local_node >= 0) {
      // multi-process siblings: every process passes only its own strips
      // (A rows [r0, r1) x K, B K x [c0, c1), C region), row-major and dense
      x.ar0 = x.ac0 = 0;
      x.ldb = x.ldc = x.c1 - x.c0;
    }
    x.K = K;
    x.cap = t->nodes[hbm[w]].capacity;
    x.kc = P.kc;
    x.pcie = t->pcie_gbs * 1e9;
    x.obm = root.bm;
    x.obn = root.bn;
    x.obk = root.bk;
    x.sched = sched;
    x.bfirst = sched == NU_SCHED_S2B ? 1 : sched == NU_SCHED_S2 ? -1 : 0;
    int use = sched == NU_SCHED_S2B ? NU_SCHED_S2 : sched;
    if (use == NU_SCHED_AUTO) {
      // P:299's row-shard reuse when the caller fixed blocks smaller than the
      // region (cfg1's 64 x 64 blocks); otherwise the C-resident schedule.
      const bool small_blocks = (root.bm > 0 && root.bm < x.r1 - x.r0) ||
                                (root.bn > 0 && root.bn < x.c1 - x.c0);
      use = small_blocks ? NU_SCHED_S1 : NU_SCHED_S2;
    }
    xs.push_back(x);
    uses.push_back(use);
  }
  // NVLink-shared staging (NEXT-1): on by default for G > 1 when every sibling
  // has a region of the same shape under S2 (opts->shared_staging < 0 disables).
  int Pr = 1, Pc = 1;
  partition_grid(G, M, N, &Pr, &Pc);
  bool share = G > 1 && !(o && o->shared_staging < 0) && t->p2p_ok && sched != NU_SCHED_S2B;
  for (int w = 0; w < G && share; ++w)
    share = uses[w] == NU_SCHED_S2 && xs[w].r1 - xs[w].r0 == xs[0].r1 - xs[0].r0 &&
            xs[w].c1 - xs[w].c0 == xs[0].c1 - xs[0].c0 && xs[w].r1 > xs[w].r0 && xs[w].c1 > xs[w].c0;
  if (share) {
    rc = build_s2_shared(B, xs, Pr, Pc, &st);
    if (rc) return rc;
  } else {
    for (int w = 0; w < G; ++w) {
      const EdgeCtx& x = xs[w];
      if (x.r1 <= x.r0 || x.c1 <= x.c0) continue;   // more GPUs than rows/cols
      rc = uses[w] == NU_SCHED_S1 ? build_s1(x, &st) : build_s2(x, &st);
      if (rc) return rc;
    }
  }
  st.ops = static_cast<int64_t>(P.ops.size());
  for (const northup_op& op : P.ops)
    if (op.op == NU_OP_COPY) st.copies++;
  return 0;
}

}  // namespace nu
