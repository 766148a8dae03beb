// HotSpot-2D over the Northup tree (S§8(f) NEXT-3; §IV-B).
//
// The paper's recursion: at level l divide the grid into
// dim(l) x dim(l) sub-blocks; move each block, its power and its four borders
// to level l+1; recurse; copy the result back.  Unrolled here for the tree
// HOST root -> HBM siblings -> SMEM leaf:
//
//   per pass (h iterations, h = the border width):
//     per block (b x b, raster order, block rows split over the siblings):
//       data_down  the window = block + h-wide borders (clipped at the grid
//                  edge) of the current grid and of P, HOST -> HBM slot
//                  (strided 2-D copies: the DMA engine gathers the east/west
//                  borders that P:317 packs by hand)
//       compute    ceil(h / 8) leaf launches ping-ponging between two window
//                  buffers of the slot; each launch's window is the previous
//                  one's valid region (shrunk by its iterations on every side
//                  that is not a grid edge)
//       data_up    the block, HBM -> the pass's output grid
//   passes alternate between Tout and a pinned scratch grid at the root so
//   the last pass writes Tout.
//
// Dependencies come from the rectangle tracker (plan_builder.h): a window of
// pass q+1 waits for the pass-q blocks it overlaps (RAW on the host grid) and
// a pass-q+1 block write waits for the pass-q windows that read that grid
// (WAR) — across siblings too (user_disjoint = false).  Three slots per
// sibling overlap H2D, compute and D2H.
#include <math.h>

#include <chrono>

#include "northup_internal.h"
#include "plan_builder.h"

namespace nu {

namespace {

inline northup_op make_stencil(int worker, int tin, int64_t tin_off, int64_t ldt, int pw,
                               int64_t pw_off, int64_t ldp, int tout, int64_t tout_off, int64_t ldo,
                               int64_t wm, int64_t wn, int64_t gy0, int64_t gx0, int64_t R,
                               int64_t C, int iters) {
  northup_op o{};
  o.op = NU_OP_STENCIL;
  o.worker = worker;
  o.stream = S_COMP;
  o.a_buf = tin;
  o.a_off = tin_off;
  o.lda = ldt;
  o.b_buf = pw;
  o.b_off = pw_off;
  o.ldb = ldp;
  o.c_buf = tout;
  o.c_off = tout_off;
  o.ldc = ldo;
  o.m = wm;
  o.n = wn;
  o.k = iters;
  o.src_off = gy0;
  o.dst_off = gx0;
  o.rows = R;
  o.cols = C;
  o.src_buf = o.dst_buf = -1;
  return o;
}

struct Win {
  int64_t y0, y1, x0, x1;   // grid coordinates, half open
};

// Valid region after `it` iterations on window w.
Win shrink(const Win& w, int it, int64_t R, int64_t C) {
  return Win{w.y0 == 0 ? 0 : w.y0 + it, w.y1 == R ? R : w.y1 - it, w.x0 == 0 ? 0 : w.x0 + it,
             w.x1 == C ? C : w.x1 - it};
}

// Emit the leaf launches of `iters` iterations on window `w`, whose cells sit
// in buffers buf[0] / buf[1] (origin (oy, ox), leading dimension ld) with
// power in `pb`; returns the buffer index holding the final values.
int emit_iterations(Builder& B, int worker, Win w, int64_t iters, int hl, const int buf[2],
                    const int64_t off[2], int pb, int64_t poff, int64_t ld, int64_t oy, int64_t ox,
                    int64_t R, int64_t C, northup_stats* st) {
  int cur = 0;
  for (int64_t done = 0; done < iters;) {
    const int it = static_cast<int>(std::min<int64_t>(hl, iters - done));
    const Win v = shrink(w, it, R, C);
    const int64_t wo = (w.y0 - oy) * ld + (w.x0 - ox), vo = (v.y0 - oy) * ld + (v.x0 - ox);
    const int64_t wm = w.y1 - w.y0, wn = w.x1 - w.x0;
    B.emit(make_stencil(worker, buf[cur], off[cur] + wo, ld, pb, poff + wo, ld, buf[cur ^ 1],
                        off[cur ^ 1] + wo, ld, wm, wn, w.y0, w.x0, R, C, it),
           {{buf[cur], off[cur] + wo, ld, wm, wn, false},
            {pb, poff + wo, ld, wm, wn, false},
            {buf[cur ^ 1], off[cur ^ 1] + vo, ld, v.y1 - v.y0, v.x1 - v.x0, true}});
    st->leaf_launches++;
    cur ^= 1;
    w = v;
    done += it;
  }
  return cur;
}

}  // namespace

int build_hotspot_plan(const northup_tree_s* t, int64_t R, int64_t C, int64_t iters,
                       const northup_hotspot_opts* o, const northup_hotspot_coeffs* k, Plan* out) {
  int rc = validate_tree(t);
  if (rc) return rc;
  if (R < 0 || C < 0 || iters < 0) return fail(NU_EINVAL, "negative grid size or iteration count");
  const int hl = o && o->leaf_iters ? o->leaf_iters : kHotspotMaxIters;
  if (hl < 1 || hl > kHotspotMaxIters)
    return fail(NU_EINVAL, "leaf_iters must be in [1, %d]", kHotspotMaxIters);
  Plan& P = *out;
  P = Plan();
  P.M = R;
  P.N = C;
  P.K = iters;
  northup_hotspot_coeffs kk{};
  if (k) kk = *k;
  else northup_hotspot_default_coeffs(R, C, &kk);
  P.hs_coef[0] = kk.cap_1;
  P.hs_coef[1] = kk.rx_1;
  P.hs_coef[2] = kk.ry_1;
  P.hs_coef[3] = kk.rz_1;
  P.hs_coef[4] = kk.amb;
  Builder B;
  B.P = &P;
  B.user_disjoint = false;
  const int T = B.add_buf(B_USER_A, 0, -1, 4ull * R * C);
  const int PW = B.add_buf(B_USER_B, 0, -1, 4ull * R * C);
  const int OUT = B.add_buf(B_USER_C, 0, -1, 4ull * R * C);
  northup_stats& st = P.stats;
  st = northup_stats{};
  const Node& root = t->nodes[0];

  if (root.storage == NU_HBM) {
    // in-HBM reference: whole-grid launches ping-ponging between Tout and an
    // arena scratch grid; the last launch writes Tout
    P.root_is_device = true;
    P.num_workers = 1;
    P.worker_node.push_back(0);
    st.num_gpus = 1;
    if (R == 0 || C == 0) return 0;
    if (iters == 0) {
      B.emit(make_copy(0, S_COMP, T, 0, C, OUT, 0, C, R, C), {{T, 0, C, R, C, false}, {OUT, 0, C, R, C, true}});
      st.bytes_d2d += 4ull * R * C;
      st.ops = static_cast<int64_t>(P.ops.size());
      return 0;
    }
    const int64_t L = (iters + hl - 1) / hl;
    const int S = L > 1 ? B.add_buf(B_ARENA, 0, 0, 4ull * R * C) : -1;
    int src = T;
    for (int64_t j = 0; j < L; ++j) {
      const int it = static_cast<int>(std::min<int64_t>(hl, iters - j * hl));
      const int dst = ((L - 1 - j) % 2 == 0) ? OUT : S;
      B.emit(make_stencil(0, src, 0, C, PW, 0, C, dst, 0, C, R, C, 0, 0, R, C, it),
             {{src, 0, C, R, C, false}, {PW, 0, C, R, C, false}, {dst, 0, C, R, C, true}});
      st.leaf_launches++;
      src = dst;
    }
    st.bm = R;
    st.bn = C;
    st.bk = hl;
    st.hbm_peak_bytes = S >= 0 ? 4ull * R * C : 0;
    st.ops = static_cast<int64_t>(P.ops.size());
    return 0;
  }
  if (root.storage != NU_HOST) return fail(NU_ENOTSUP, "HotSpot-2D needs a HOST or HBM root");
  std::vector<int> hbm;
  for (int c : root.children) {
    if (t->nodes[c].storage != NU_HBM)
      return fail(NU_ENOTSUP, "HOST root children must be HBM nodes (node %d is not)", c);
    hbm.push_back(c);
  }
  if (hbm.empty()) return fail(NU_EINVAL, "HOST root has no HBM child");
  if (t->local_node >= 0) return fail(NU_ENOTSUP, "HotSpot-2D runs in one process (no set_local)");
  const int G = static_cast<int>(hbm.size());
  P.num_workers = G;
  P.worker_node = hbm;
  st.num_gpus = G;
  if (R == 0 || C == 0) return 0;
  if (iters == 0) {
    B.emit(make_copy(0, S_D2H, T, 0, C, OUT, 0, C, R, C), {{T, 0, C, R, C, false}, {OUT, 0, C, R, C, true}});
    st.ops = static_cast<int64_t>(P.ops.size());
    return 0;
  }
  uint64_t cap = 0;
  for (int h : hbm)
    if (t->nodes[h].capacity) cap = cap ? std::min(cap, t->nodes[h].capacity) : t->nodes[h].capacity;
  constexpr int kS = kSlots;
  constexpr int kRowBands = 3;   // row-band staging buffers per sibling (T and P, full grid width)
  // slot footprint: three windows (temperature ping, pong, power), (b + 2h) square
  // slots of three windows (temperature ping, pong, power), (b + 2h) square,
  // plus two staging strips (window rows x 2h) for the temperature columns a
  // window shares with the next one (see below)
  auto arena_bytes = [&](int64_t b, int64_t h) {
    const int64_t W = std::min(b + 2 * h, std::max(R, C));
    return 4ull * kS * 3 * static_cast<uint64_t>(std::min(W, R)) * pad_ld(std::min(W, C)) +
           4ull * 2 * static_cast<uint64_t>(std::min(W, R)) * pad_ld(2 * h);
  };
  // the row-band buffers (full grid width) come on top, only when they fit
  auto band_bytes = [&](int64_t h) { return 4ull * kRowBands * 2 * static_cast<uint64_t>(2 * h) * pad_ld(C); };
  const int64_t edge = std::max(R, C);
  int64_t b = o && o->block > 0 ? o->block : std::min<int64_t>(edge, 8192);   // P:325 8k blocking
  int64_t h = o && o->halo > 0 ? o->halo : 0;
  if (h <= 0) {
    // iterations per visit: all of them when the border overhead stays small,
    // else a multiple of the leaf's iterations with <= ~15% extra window area
    const int64_t hmax = std::max<int64_t>(hl, (static_cast<int64_t>(0.035 * b) / hl) * hl);
    h = std::min(iters, hmax);
  }
  h = std::min(h, iters);
  if (!(o && o->block > 0)) {
    while (cap && arena_bytes(b, h) > cap && b > 8) b = b > 64 ? rup(b / 2, 64) : std::max<int64_t>(8, b / 2);
    // equal blocks: the fewest blocks of at most b cells per side
    const int64_t g = b >= 64 ? 64 : 8;
    const int64_t nby = cdiv(R, b), nbx = cdiv(C, b);
    const int64_t be = std::max(rup(cdiv(R, nby), g), rup(cdiv(C, nbx), g));
    if (!cap || arena_bytes(std::min(be, edge), h) <= cap) b = std::min(be, edge);
  }
  if (cap && arena_bytes(b, h) > cap)
    return fail(NU_ENOMEM, "HBM capacity %llu B below the HotSpot block %lld + border %lld",
                (unsigned long long)cap, (long long)b, (long long)h);
  const int64_t W = std::min(b + 2 * h, edge);
  const int64_t WR = std::min(W, R), LD = pad_ld(std::min(W, C));
  const int64_t win = WR * LD;   // elements per window buffer
  std::vector<int> arena(G);
  const bool use_bands = !cap || arena_bytes(b, h) + band_bytes(h) <= cap;
  const uint64_t abytes = arena_bytes(b, h) + (use_bands ? band_bytes(h) : 0);
  for (int w = 0; w < G; ++w) arena[w] = B.add_buf(B_ARENA, hbm[w], w, abytes);
  const int64_t Q = cdiv(iters, h);
  const int S = Q > 1 ? B.add_buf(B_DRAM, 0, -1, 4ull * R * C) : -1;   // pinned scratch grid
  const int64_t nby = cdiv(R, b), nbx = cdiv(C, b);
  st.bm = st.bn = b;
  st.bk = h;
  st.hbm_peak_bytes = abytes;
  std::vector<int64_t> slot_ctr(G, 0);
  // Each sibling's previous window of the same pass: a window that shares its
  // rows takes the power columns it has in common with it from that window's
  // slot (a device copy) instead of over PCIe again (2h columns per block; P is
  // read-only, unlike the temperature windows, which the iterations overwrite).
  struct PrevWin {
    bool valid = false;
    int64_t q = -1, y0 = 0, y1 = 0, x0 = 0, x1 = 0, poff = 0;
  };
  std::vector<PrevWin> prevw(G);
  // The temperature columns two such windows share are copied out of the
  // earlier window (into one of two staging strips after its slot is loaded,
  // before its second launch overwrites them) and into the later one, so they
  // do not cross PCIe twice either.
  const int64_t SLD = pad_ld(2 * h);                                // staging strip leading dimension
  const int64_t stg0 = static_cast<int64_t>(kS) * 3 * win;          // first strip (elements)
  std::vector<int> stg_next(G, 0);                                  // strip the next hand-off uses
  std::vector<int> stg_have(G, -1);                                 // strip holding the hand-off for the next window
  // Row bands: the 2 itq rows a window shares with the sibling's window below
  // it (same pass, same columns or a subset) are copied, T and P, into a
  // full-width band buffer after the upper window lands (before its second
  // launch overwrites T) and from there into the lower window.
  const int64_t LDC = pad_ld(C), rs0 = stg0 + 2 * WR * SLD;
  auto rs_t = [&](int buf) { return rs0 + static_cast<int64_t>(buf) * 2 * (2 * h) * LDC; };
  auto rs_p = [&](int buf) { return rs_t(buf) + (2 * h) * LDC; };
  struct Band {
    int64_t row = -1, q = -1;
    int buf = -1;
    std::vector<std::pair<int64_t, int64_t>> cov;   // grid columns staged so far
    bool covers(int64_t x0, int64_t x1) const {
      int64_t at = x0;   // intervals arrive left to right per block row
      for (bool grew = true; grew && at < x1;) {
        grew = false;
        for (const auto& c : cov)
          if (c.first <= at && c.second > at) {
            at = c.second;
            grew = true;
          }
      }
      return at >= x1;
    }
  };
  std::vector<std::vector<Band>> bands(G);
  std::vector<int> rs_next(G, 0);
  auto window_of = [&](const Win& blk, int64_t itq) {
    return Win{std::max<int64_t>(0, blk.y0 - itq), std::min(R, blk.y1 + itq), std::max<int64_t>(0, blk.x0 - itq),
               std::min(C, blk.x1 + itq)};
  };
  int src = T;
  for (int64_t q = 0; q < Q; ++q) {
    const int64_t itq = std::min(h, iters - q * h);
    const int dst = ((Q - 1 - q) % 2 == 0) ? OUT : S;
    const int ldg_src = C, ldg_dst = C;
    // Blocks of one pass are independent (they read the pass's source grid and
    // write its destination), so each sibling's first block of the first pass and
    // last block of the last pass are split 2 x 2: the pipeline fills after a
    // quarter-size window and drains a quarter-size block (a little more border
    // recomputation on those two blocks only).
    for (auto& bl : bands) bl.clear();
    std::vector<Win> blks;
    std::vector<int> owner;
    for (int64_t by = 0; by < nby; ++by) {
      const int w = static_cast<int>(by * G / nby);   // block rows split over the siblings
      const bool w_first_row = by == 0 || static_cast<int>((by - 1) * G / nby) != w;
      const bool w_last_row = by == nby - 1 || static_cast<int>((by + 1) * G / nby) != w;
      for (int64_t bx = 0; bx < nbx; ++bx) {
        const Win blk{by * b, std::min(R, (by + 1) * b), bx * b, std::min(C, (bx + 1) * b)};
        const bool split = ((q == 0 && w_first_row && bx == 0) || (q == Q - 1 && w_last_row && bx == nbx - 1)) &&
                           blk.y1 - blk.y0 >= 256 && blk.x1 - blk.x0 >= 256;
        if (!split) {
          blks.push_back(blk);
          owner.push_back(w);
          continue;
        }
        const int64_t ym = blk.y0 + rup(cdiv(blk.y1 - blk.y0, 2), 64), xm = blk.x0 + rup(cdiv(blk.x1 - blk.x0, 2), 64);
        for (const Win& sb : {Win{blk.y0, ym, blk.x0, xm}, Win{blk.y0, ym, xm, blk.x1}, Win{ym, blk.y1, blk.x0, xm},
                              Win{ym, blk.y1, xm, blk.x1}}) {
          blks.push_back(sb);
          owner.push_back(w);
        }
      }
    }
    for (size_t bi = 0; bi < blks.size(); ++bi) {
      const int w = owner[bi];
      {
        const Win blk = blks[bi];
        const Win win_g = window_of(blk, itq);
        const int64_t wm = win_g.y1 - win_g.y0, wn = win_g.x1 - win_g.x0;
        const int sl = static_cast<int>(slot_ctr[w]++ % kS);
        const int64_t base = static_cast<int64_t>(sl) * 3 * win;
        const int64_t off[2] = {base, base + win};
        const int64_t poff = base + 2 * win;
        const int bufs[2] = {arena[w], arena[w]};
        // data_down: window of the current grid and of P (block + borders).
        // Rows [0, r_lo) may come from a row band, columns [0, tc0) / [0, pc0)
        // of the other rows from the sibling's previous window; the rest over PCIe.
        const int64_t bh = 2 * itq;
        int64_t r_lo = 0;
        if (use_bands && win_g.y0 > 0 && wm > bh) {
          for (const Band& bd : bands[w])
            if (bd.q == q && bd.row == win_g.y0 && bd.covers(win_g.x0, win_g.x1)) {
              r_lo = bh;
              B.emit(make_copy(w, S_D2D, arena[w], rs_t(bd.buf) + win_g.x0, LDC, arena[w], off[0], LD, bh, wn),
                     {{arena[w], rs_t(bd.buf) + win_g.x0, LDC, bh, wn, false}, {arena[w], off[0], LD, bh, wn, true}});
              B.emit(make_copy(w, S_D2D, arena[w], rs_p(bd.buf) + win_g.x0, LDC, arena[w], poff, LD, bh, wn),
                     {{arena[w], rs_p(bd.buf) + win_g.x0, LDC, bh, wn, false}, {arena[w], poff, LD, bh, wn, true}});
              st.bytes_d2d += 8ull * bh * wn;
              break;
            }
        }
        const int64_t rm = wm - r_lo;                                  // rows not from a band
        const int64_t go = (win_g.y0 + r_lo) * C + win_g.x0;
        const int64_t to = off[0] + r_lo * LD, po = poff + r_lo * LD;   // their start in the slot
        const PrevWin& pv = prevw[w];
        const bool shares = pv.valid && pv.q == q && pv.y0 == win_g.y0 && pv.y1 == win_g.y1 && pv.x0 < win_g.x0 &&
                            pv.x1 > win_g.x0;
        const int64_t ov = shares ? std::min(pv.x1, win_g.x1) - win_g.x0 : 0;   // shared columns
        int64_t tc0 = 0;   // T columns [0, tc0) of those rows come from a staging strip
        if (shares && stg_have[w] >= 0 && ov <= 2 * h) {
          tc0 = ov;
          const int64_t so = stg0 + static_cast<int64_t>(stg_have[w]) * WR * SLD + r_lo * SLD;
          B.emit(make_copy(w, S_D2D, arena[w], so, SLD, arena[w], to, LD, rm, tc0),
                 {{arena[w], so, SLD, rm, tc0, false}, {arena[w], to, LD, rm, tc0, true}});
          st.bytes_d2d += 4ull * rm * tc0;
        }
        stg_have[w] = -1;
        if (wn > tc0)
          B.emit(make_copy(w, S_H2D, src, go + tc0, ldg_src, arena[w], to + tc0, LD, rm, wn - tc0),
                 {{src, go + tc0, ldg_src, rm, wn - tc0, false}, {arena[w], to + tc0, LD, rm, wn - tc0, true}});
        int64_t pc0 = 0;   // P columns [0, pc0) of those rows come from the previous window's slot
        if (shares) {
          pc0 = ov;
          const int64_t so = pv.poff + r_lo * LD + (win_g.x0 - pv.x0);
          B.emit(make_copy(w, S_D2D, arena[w], so, LD, arena[w], po, LD, rm, pc0),
                 {{arena[w], so, LD, rm, pc0, false}, {arena[w], po, LD, rm, pc0, true}});
          st.bytes_d2d += 4ull * rm * pc0;
        }
        if (wn > pc0)
          B.emit(make_copy(w, S_H2D, PW, go + pc0, C, arena[w], po + pc0, LD, rm, wn - pc0),
                 {{PW, go + pc0, C, rm, wn - pc0, false}, {arena[w], po + pc0, LD, rm, wn - pc0, true}});
        st.bytes_h2d += 4ull * rm * (wn - tc0) + 4ull * rm * (wn - pc0);
        // hand the columns this window shares with the sibling's next window
        // (same pass, same rows) to a staging strip before the iterations
        // overwrite them
        if (bi + 1 < blks.size() && owner[bi + 1] == w) {
          const Win nx = window_of(blks[bi + 1], itq);
          const int64_t ovn = nx.y0 == win_g.y0 && nx.y1 == win_g.y1 && nx.x0 > win_g.x0 && nx.x0 < win_g.x1
                                  ? std::min(win_g.x1, nx.x1) - nx.x0 : 0;
          if (ovn > 0 && ovn <= 2 * h) {
            const int sidx = stg_next[w];
            stg_next[w] ^= 1;
            const int64_t so = off[0] + (nx.x0 - win_g.x0), dso = stg0 + static_cast<int64_t>(sidx) * WR * SLD;
            B.emit(make_copy(w, S_D2D, arena[w], so, LD, arena[w], dso, SLD, wm, ovn),
                   {{arena[w], so, LD, wm, ovn, false}, {arena[w], dso, SLD, wm, ovn, true}});
            st.bytes_d2d += 4ull * wm * ovn;
            stg_have[w] = sidx;
          }
        }
        // and the rows it shares with a later window of the sibling below it
        if (use_bands && win_g.y1 < R && wm > bh) {
          const int64_t brow = win_g.y1 - bh;
          bool needed = false;
          for (size_t bj = bi + 1; bj < blks.size() && !needed; ++bj) {
            if (owner[bj] != w) continue;
            const Win lw = window_of(blks[bj], itq);
            needed = lw.y0 == brow && lw.x0 < win_g.x1 && lw.x1 > win_g.x0;
          }
          if (needed) {
            Band* bd = nullptr;
            for (Band& x : bands[w])
              if (x.q == q && x.row == brow) bd = &x;
            if (!bd) {
              const int buf = rs_next[w];
              rs_next[w] = (rs_next[w] + 1) % kRowBands;
              auto& bl = bands[w];
              bl.erase(std::remove_if(bl.begin(), bl.end(), [&](const Band& x) { return x.buf == buf; }), bl.end());
              bl.push_back(Band{brow, q, buf, {}});
              bd = &bl.back();
            }
            const int64_t tso = off[0] + (wm - bh) * LD, pso = poff + (wm - bh) * LD;
            B.emit(make_copy(w, S_D2D, arena[w], tso, LD, arena[w], rs_t(bd->buf) + win_g.x0, LDC, bh, wn),
                   {{arena[w], tso, LD, bh, wn, false}, {arena[w], rs_t(bd->buf) + win_g.x0, LDC, bh, wn, true}});
            B.emit(make_copy(w, S_D2D, arena[w], pso, LD, arena[w], rs_p(bd->buf) + win_g.x0, LDC, bh, wn),
                   {{arena[w], pso, LD, bh, wn, false}, {arena[w], rs_p(bd->buf) + win_g.x0, LDC, bh, wn, true}});
            st.bytes_d2d += 8ull * bh * wn;
            bd->cov.emplace_back(win_g.x0, win_g.x1);
          }
        }
        prevw[w] = PrevWin{true, q, win_g.y0, win_g.y1, win_g.x0, win_g.x1, poff};
        const int fin = emit_iterations(B, w, win_g, itq, hl, bufs, off, arena[w], poff, LD, win_g.y0,
                                        win_g.x0, R, C, &st);
        // data_up: the block
        const int64_t bo = off[fin] + (blk.y0 - win_g.y0) * LD + (blk.x0 - win_g.x0);
        const int64_t bm = blk.y1 - blk.y0, bn = blk.x1 - blk.x0;
        const int64_t dgo = blk.y0 * C + blk.x0;
        B.emit(make_copy(w, S_D2H, arena[w], bo, LD, dst, dgo, ldg_dst, bm, bn),
               {{arena[w], bo, LD, bm, bn, false}, {dst, dgo, ldg_dst, bm, bn, true}});
        st.bytes_d2h += 4ull * bm * bn;
      }
    }
    src = dst;
  }
  st.ops = static_cast<int64_t>(P.ops.size());
  for (const northup_op& op : P.ops)
    if (op.op == NU_OP_COPY) st.copies++;
  return B.overflow ? fail(NU_ENOTSUP, "dependency fan-in above 16") : 0;
}

}  // namespace nu

using namespace nu;

extern "C" {

int northup_hotspot_default_coeffs(int64_t rows, int64_t cols, northup_hotspot_coeffs* out) {
  if (!out) return fail(NU_EINVAL, "NULL argument");
  (void)rows;
  (void)cols;
  // [18]'s chip model (RH1) at its 1024-cell pitch (RH2): 16 mm / 1024
  const double t_chip = 0.0005, k_si = 100.0, spec_heat = 1.75e6, factor = 0.5;
  const double max_pd = 3.0e6, precision = 0.001, pitch = 0.016 / 1024.0;
  const double cap = factor * spec_heat * t_chip * pitch * pitch;
  const double rx = pitch / (2.0 * k_si * t_chip * pitch);
  const double ry = pitch / (2.0 * k_si * t_chip * pitch);
  const double rz = t_chip / (k_si * pitch * pitch);
  const double step = precision / (max_pd / (factor * t_chip * spec_heat));
  out->cap_1 = static_cast<float>(step / cap);
  out->rx_1 = static_cast<float>(1.0 / rx);
  out->ry_1 = static_cast<float>(1.0 / ry);
  out->rz_1 = static_cast<float>(1.0 / rz);
  out->amb = 80.0f;
  return 0;
}

int northup_hotspot_leaf(const float* tin, int64_t ldt, const float* pw, int64_t ldp, float* tout,
                         int64_t ldo, int64_t wm, int64_t wn, int64_t gy0, int64_t gx0,
                         int64_t rows, int64_t cols, int iters, const northup_hotspot_coeffs* k,
                         void* stream) {
  northup_hotspot_coeffs kk{};
  if (k) kk = *k;
  else northup_hotspot_default_coeffs(rows, cols, &kk);
  const float coef[5] = {kk.cap_1, kk.rx_1, kk.ry_1, kk.rz_1, kk.amb};
  return hotspot_launch(tin, ldt, pw, ldp, tout, ldo, wm, wn, gy0, gx0, rows, cols, iters, coef,
                        static_cast<cudaStream_t>(stream));
}

int northup_hotspot_plan(northup_tree_t t, int64_t rows, int64_t cols, int64_t iters,
                         const northup_hotspot_opts* opts, northup_plan_t* out) {
  if (!t || !out) return fail(NU_EINVAL, "NULL argument");
  northup_plan_s* p = new northup_plan_s();
  int rc = build_hotspot_plan(t, rows, cols, iters, opts, nullptr, &p->plan);
  if (rc) {
    delete p;
    return rc;
  }
  *out = p;
  return 0;
}

int northup_hotspot(northup_tree_t t, northup_buf_t T, northup_buf_t P, northup_buf_t Tout,
                    int64_t rows, int64_t cols, int64_t iters, const northup_hotspot_coeffs* k,
                    const northup_hotspot_opts* opts, northup_stats* s) {
  const auto t0 = std::chrono::steady_clock::now();
  if (!t || !T || !P || !Tout) return fail(NU_EINVAL, "NULL argument");
  if (!t->finalized) return fail(NU_ESTATE, "tree not finalized");
  if (t->busy) return fail(NU_ESTATE, "a call is already in flight on this tree");
  if (T->tree != t || P->tree != t || Tout->tree != t) return fail(NU_EINVAL, "buffer from another tree");
  if (T->node != 0 || P->node != 0 || Tout->node != 0)
    return fail(NU_EINVAL, "T, P and Tout must live at the root node");
  if (rows < 0 || cols < 0 || iters < 0) return fail(NU_EINVAL, "negative argument");
  const uint64_t need = 4ull * rows * cols;
  if (T->bytes < need || P->bytes < need || Tout->bytes < need)
    return fail(NU_EINVAL, "buffer smaller than the grid");
  if (T == Tout || T->ptr == Tout->ptr) return fail(NU_EINVAL, "T and Tout must differ");
  northup_stats local{};
  northup_stats* st = s ? s : &local;
  *st = northup_stats{};
  t->busy = true;
  Plan plan;
  int rc = build_hotspot_plan(t, rows, cols, iters, opts, k, &plan);
  if (!rc) {
    *st = plan.stats;
    st->t_plan_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    northup_gemm_opts go{};
    go.collect_timing = opts ? opts->collect_timing : 0;
    go.shared_staging = -1;
    int prev = 0;
    cudaGetDevice(&prev);
    rc = execute_plan(t, plan, T, P, Tout, &go, st);
    cudaSetDevice(prev);
  }
  t->busy = false;
  st->t_total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return rc;
}

}  // extern "C"
