// fold.cpp -- host construction of the stage-folded schedule of the persistent
// forward (DESIGN.md §4 "stage folding").
//
// A pin p with exactly one fanin arc e' = (j -> p) and exactly one fanout arc
// e = (p -> q) that is not an endpoint -- in a netlist, a cell input pin -- is
// "folded": its arrival (a merge of the candidates of e' alone, Alg 1 with one
// fanin) is computed inside the item of its sink q, in registers, right before
// q's candidates over e are formed.  p is still written to the state arrays, so
// every consumer of the per-pin state (slack, backward, incremental pass,
// arrivals) sees exactly what the per-level schedule writes; the arithmetic per
// pin is the same device code, so the results are bit-identical.  What changes
// is the dependency depth: q waits for j, not for p, so a (net arc, cell arc)
// pair costs one level-to-level step instead of two (162 -> ~82 steps at C4).
//
// Rule (canonical order): p is folded iff indeg(p) = 1, outdeg(p) = 1, p is
// not an endpoint, and the source j of its fanin arc is not folded.  Then the
// sink q of p is never folded either (its fanin source p is), so folding never
// nests.  Every other pin is a "head".  Heads are scheduled by super-level:
// slevel = 0 for indeg-0 pins, else 1 + max over its fanin arcs (p -> q) of
// slevel(p) (p a head) or slevel(j) (p folded, j its source); heads are
// ordered by slevel, then (past level 0) by shape (fanin count, folded
// entries, non-unate arc), then canonical position, so the startpoints keep
// positions 0..num_src-1.
#include <algorithm>

#include <vector_functions.h>

#include "internal.h"

namespace insta {

void build_fold(const HostLevels& h, const std::vector<int32_t>& fin_src, const std::vector<float4>& fin_ms,
                const std::vector<int32_t>& ep_of_pin, const std::vector<int32_t>& lfo_ptr,
                const std::vector<int32_t>& lfo, const std::vector<int32_t>& heavy_slot, int grid, FoldHost* out) {
  FoldHost& f = *out;
  f = FoldHost();
  const int32_t n = h.n;
  const auto& fp = h.fanin_ptr;
  const auto& op = h.fanout_ptr;
  f.folded.assign(size_t(n), 0);
  for (int32_t p = 0; p < n; ++p) {
    if (fp[p + 1] - fp[p] != 1 || op[p + 1] - op[p] != 1 || ep_of_pin[p] >= 0) continue;
    const int32_t j = fin_src[fp[p]] & kSrcMask;
    if (!f.folded[j]) f.folded[p] = 1;
  }
  // super-levels of heads (canonical order is topological)
  std::vector<int32_t> sl(size_t(n), 0);
  int32_t max_sl = 0;
  for (int32_t q = 0; q < n; ++q) {
    if (f.folded[q] || fp[q + 1] == fp[q]) continue;
    int32_t s = 0;
    for (int32_t x = fp[q]; x < fp[q + 1]; ++x) {
      int32_t p = fin_src[x] & kSrcMask;
      if (f.folded[p]) p = fin_src[fp[p]] & kSrcMask;
      s = std::max(s, sl[p] + 1);
    }
    sl[q] = s;
    max_sl = std::max(max_sl, s);
  }
  const int32_t SL = n > 0 ? max_sl + 1 : 0;
  f.slevel_ptr.assign(size_t(SL) + 1, 0);
  for (int32_t q = 0; q < n; ++q)
    if (!f.folded[q]) ++f.slevel_ptr[sl[q] + 1];
  for (int32_t s = 0; s < SL; ++s) f.slevel_ptr[s + 1] += f.slevel_ptr[s];
  const int32_t H = SL > 0 ? f.slevel_ptr[SL] : 0;
  f.hd_pin.assign(size_t(H), 0);
  {
    std::vector<int32_t> fill(f.slevel_ptr.begin(), f.slevel_ptr.end() - (SL > 0 ? 1 : 0));
    for (int32_t q = 0; q < n; ++q)
      if (!f.folded[q]) f.hd_pin[fill[sl[q]]++] = q;
  }
  // within a super-level (past the startpoints) heads are ordered by their
  // shape -- fanin count, folded entries, a non-unate arc -- then canonical
  // position: the heads of one level are independent, and a warp of
  // same-shape heads runs the fanin-specialized code without divergence
  // (sweep.cu); every schedule walks the same head order
  {
    std::vector<int64_t> key(size_t(n), 0);
    for (int32_t q = 0; q < n; ++q) {
      if (f.folded[q]) continue;
      const int32_t nf = fp[q + 1] - fp[q];
      int32_t nfold = 0, non = 0;
      for (int32_t x = fp[q]; x < fp[q + 1]; ++x) {
        const int32_t p = fin_src[x] & kSrcMask;
        if (uint32_t(fin_src[x]) >> kUnateShift == 2) non = 1;
        if (f.folded[p]) {
          ++nfold;
          if (uint32_t(fin_src[fp[p]]) >> kUnateShift == 2) non = 1;
        }
      }
      key[q] = (int64_t(std::min(nf, 255)) << 40) | (int64_t(std::min(nfold, 255)) << 32) | (int64_t(non) << 31) | q;
    }
    // sorted within each CTA slice of the sweep (sweep.cu cta_slice: CTA c of G
    // owns heads [lo + n c / G, lo + n (c + 1) / G) of a level): every CTA keeps
    // the level's natural mix of shapes (balanced work), its warps get uniform ones
    const int64_t G = std::max(grid, 1);
    for (int32_t s = 1; s < SL; ++s) {
      const int64_t lo = f.slevel_ptr[s], nh = f.slevel_ptr[s + 1] - lo;
      for (int64_t c = 0; c < G; ++c)
        std::sort(f.hd_pin.begin() + lo + nh * c / G, f.hd_pin.begin() + lo + nh * (c + 1) / G,
                  [&](int32_t x, int32_t y) { return key[x] < key[y]; });
    }
  }
  // entries: one per fanin arc of a head, in fanin row order
  f.hd_ptr.assign(size_t(H) + 1, 0);
  f.hd_q0.assign(size_t(H), 0);
  f.hd_nfold.assign(size_t(H), 0);
  const int64_t X = h.e - std::count(f.folded.begin(), f.folded.end(), uint8_t(1));
  f.ext_w.assign(size_t(X), 0);
  f.ext_f.assign(size_t(X), 0);
  f.ext_fq.assign(size_t(X), -1);
  f.ext_ms.assign(size_t(X), make_float4(0.f, 0.f, 0.f, 0.f));
  f.ext_fms.assign(size_t(X), make_float4(0.f, 0.f, 0.f, 0.f));
  f.arc_xpos.assign(size_t(h.e), -1);
  f.ext_qpos.assign(size_t(X), 0);
  f.ext_bw.assign(size_t(X), 0);
  f.ext_arc.assign(size_t(X), 0);
  f.ext_farc.assign(size_t(X), -1);
  f.ext_h.assign(size_t(X), 0);
  f.hd_hslot.assign(size_t(H), -1);
  f.hd_eop.assign(size_t(H), -1);
  f.hlfo_ptr.assign(size_t(H) + 1, 0);
  f.hlfo.clear();
  f.ep_head.assign(size_t(std::count_if(ep_of_pin.begin(), ep_of_pin.end(), [](int32_t v) { return v >= 0; })), -1);
  int64_t x = 0;
  for (int32_t hh = 0; hh < H; ++hh) {
    const int32_t q = f.hd_pin[hh];
    f.hd_q0[hh] = fp[q];
    f.hd_hslot[hh] = heavy_slot[q];
    if (ep_of_pin[q] >= 0) f.ep_head[ep_of_pin[q]] = hh;
    f.hd_eop[hh] = ep_of_pin[q];
    for (int32_t r = lfo_ptr[q]; r < lfo_ptr[q + 1]; ++r) f.hlfo.push_back(lfo[r]);
    f.hlfo_ptr[hh + 1] = int32_t(f.hlfo.size());
    for (int32_t y = fp[q]; y < fp[q + 1]; ++y, ++x) {
      const int32_t p = fin_src[y] & kSrcMask;
      const int32_t u = int32_t(uint32_t(fin_src[y]) >> kUnateShift);
      f.ext_ms[x] = fin_ms[y];
      f.arc_xpos[h.fanin_arc[y]] = int32_t(2 * x);
      f.ext_qpos[x] = y;
      f.ext_h[x] = hh;
      f.ext_arc[x] = h.fanin_arc[y];
      f.ext_bw[x] = fin_src[y];
      if (f.folded[p]) {
        const int32_t y2 = fp[p];
        const int32_t j = fin_src[y2] & kSrcMask;
        const int32_t u2 = int32_t(uint32_t(fin_src[y2]) >> kUnateShift);
        f.ext_w[x] = j | (1 << kFoldBit) | int32_t(uint32_t(u) << kUnateShift);
        f.ext_f[x] = p | int32_t(uint32_t(u2) << kUnateShift);
        f.ext_fq[x] = y2;
        f.ext_fms[x] = fin_ms[y2];
        f.arc_xpos[h.fanin_arc[y2]] = int32_t(2 * x + 1);
        f.ext_farc[x] = h.fanin_arc[y2];
        f.ext_bw[x] = fin_src[y2];
        ++f.hd_nfold[hh];
      } else {
        f.ext_w[x] = p | int32_t(uint32_t(u) << kUnateShift);
      }
    }
    f.hd_ptr[hh + 1] = int32_t(x);
  }
  // level-synchronous sweep: source head of every entry and the consumer
  // heads of every head (the heads whose entries read its record)
  std::vector<int32_t> head_of(size_t(n), -1);
  for (int32_t hh = 0; hh < H; ++hh) head_of[f.hd_pin[hh]] = hh;
  f.ext_sh.assign(size_t(X), -1);
  std::vector<int64_t> pair_src;
  std::vector<int32_t> pair_dst;
  pair_src.reserve(size_t(X));
  pair_dst.reserve(size_t(X));
  for (int32_t hh = 0; hh < H; ++hh) {
    for (int32_t y = f.hd_ptr[hh]; y < f.hd_ptr[hh + 1]; ++y) {
      const int32_t sp = f.ext_w[y] & kSrcMask;
      f.ext_sh[y] = head_of[sp];
      pair_src.push_back(head_of[sp]);
      pair_dst.push_back(hh);
    }
  }
  // cone pass (sweep.cu): consumer heads of every head (deduplicated rows,
  // marked by a changed head when short), their super-level range (flagged
  // when the row is long), and per head whether one of its sources has a long
  // row (such a head checks its sources' change stamps itself)
  f.hfo_ptr.assign(size_t(H) + 1, 0);
  for (int64_t k : pair_src) ++f.hfo_ptr[k + 1];
  for (int32_t hh = 0; hh < H; ++hh) f.hfo_ptr[hh + 1] += f.hfo_ptr[hh];
  f.hfo.assign(pair_src.size(), 0);
  {
    std::vector<int32_t> fill(f.hfo_ptr.begin(), f.hfo_ptr.end() - 1);
    for (size_t k = 0; k < pair_src.size(); ++k) f.hfo[fill[pair_src[k]]++] = pair_dst[k];
    int32_t w = 0, lo = 0;
    for (int32_t hh = 0; hh < H; ++hh) {
      const int32_t hi = f.hfo_ptr[hh + 1];
      std::sort(f.hfo.begin() + lo, f.hfo.begin() + hi);
      const int32_t start = w;
      for (int32_t k = lo; k < hi; ++k)
        if (k == lo || f.hfo[k] != f.hfo[k - 1]) f.hfo[w++] = f.hfo[k];
      f.hfo_ptr[hh] = start;
      lo = hi;
    }
    f.hfo_ptr[H] = w;
    f.hfo.resize(size_t(w));
  }
  f.hd_csl.assign(size_t(H), -1);
  f.hd_hsrc.assign(size_t(H), 0);
  for (int32_t hh = 0; hh < H; ++hh) {
    const int32_t r0 = f.hfo_ptr[hh], r1 = f.hfo_ptr[hh + 1];
    if (r1 == r0) continue;
    int32_t cmin = INT32_MAX, cmax = -1;
    for (int32_t r = r0; r < r1; ++r) {
      const int32_t cs = sl[f.hd_pin[f.hfo[r]]];
      cmin = std::min(cmin, cs);
      cmax = std::max(cmax, cs);
    }
    f.hd_csl[hh] = std::min(cmin, 65535) | (std::min(cmax, 65535) << 16);
    if (r1 - r0 > kConeRow)
      for (int32_t r = r0; r < r1; ++r) f.hd_hsrc[f.hfo[r]] = 1;
  }
  // incremental pass: the head whose item evaluates each arc
  f.arc_head.assign(size_t(h.e), -1);
  for (int32_t hh = 0; hh < H; ++hh) {
    for (int32_t y = f.hd_ptr[hh]; y < f.hd_ptr[hh + 1]; ++y) {
      f.arc_head[f.ext_arc[y]] = hh;
      if (f.ext_farc[y] >= 0) f.arc_head[f.ext_farc[y]] = hh;
    }
  }
}

}  // namespace insta
