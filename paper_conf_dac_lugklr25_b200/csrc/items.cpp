// items.cpp -- host construction of the per-CTA work items of the persistent
// level-slice kernels.
//
// Each timing level is cut into rounds x G contiguous chunks of (nearly) equal
// work, G = number of resident CTAs.  Work of a pin is 1 + its fanin arcs
// (forward) or 1 + fanin arcs + light fanout entries (backward).  The number of
// rounds doubles until every chunk fits the shared-memory stage of one item; a
// single pin that can never fit is flagged "direct" (topology read from global).
#include <algorithm>

#include <vector_functions.h>

#include "internal.h"

namespace insta {
namespace {

struct Caps {
  int64_t pins, arcs, fanout;
};

// Cut pins [lo, hi) into n chunks by work quantiles; returns n+1 boundaries.
void quantile_cuts(const std::vector<int64_t>& prefix /* over [lo, hi], prefix[0] = 0 */,
                   int32_t lo, int64_t n, std::vector<int32_t>* cuts) {
  const int64_t W = prefix.back();
  cuts->assign(size_t(n) + 1, lo);
  (*cuts)[n] = lo + int32_t(prefix.size() - 1);
  for (int64_t j = 1; j < n; ++j) {
    // first pin index k such that prefix[k] >= j*W/n (integer ceil)
    const int64_t target = (j * W + n - 1) / n;
    const int64_t k = std::lower_bound(prefix.begin(), prefix.end(), target) - prefix.begin();
    (*cuts)[j] = lo + int32_t(std::min<int64_t>(k, int64_t(prefix.size() - 1)));
  }
  for (int64_t j = 1; j <= n; ++j) (*cuts)[j] = std::max((*cuts)[j], (*cuts)[j - 1]);
}

// Cut every level (unit ranges [lptr[l], lptr[l+1]) of a level-ordered unit
// array, forward or reverse level order) into rounds x G balanced chunks.
// work(u): work of unit u; over(a, b): chunk [a, b) exceeds the stage caps;
// emit(T, l, a, b, flags): append the item.
template <class Work, class Over, class Emit>
void cut_levels(ItemTable& T, int G, const std::vector<int32_t>& lptr, bool reverse, Work&& work, Over&& over,
                Emit&& emit) {
  const int L = int(lptr.size()) - 1;
  T = ItemTable();
  T.level_step0.assign(size_t(std::max(L, 0)), 0);
  T.level_steps.assign(size_t(std::max(L, 0)), 0);
  std::vector<int64_t> prefix;
  std::vector<int32_t> cuts;
  for (int li = 0; li < L; ++li) {
    const int l = reverse ? (L - 1 - li) : li;
    const int32_t lo = lptr[l], hi = lptr[l + 1];
    prefix.assign(size_t(hi - lo) + 1, 0);
    for (int32_t p = lo; p < hi; ++p) prefix[p - lo + 1] = prefix[p - lo] + work(p);
    int64_t m = 1;
    for (;;) {
      quantile_cuts(prefix, lo, m * G, &cuts);
      bool ok = true;
      for (int64_t j = 0; j < m * G && ok; ++j) {
        const int32_t a = cuts[j], b = cuts[j + 1];
        if (b - a <= 1) continue;   // single units are always accepted (direct if too big)
        if (over(a, b)) ok = false;
      }
      if (ok || m * G >= int64_t(hi - lo)) break;
      m *= 2;
    }
    // with m*G >= units every chunk holds <= 1 unit, so the loop above terminates
    T.level_step0[l] = T.num_steps;
    T.level_steps[l] = int32_t(m);
    for (int64_t r = 0; r < m; ++r) {
      for (int c = 0; c < G; ++c) {
        const int64_t j = r * G + c;
        const int32_t a = cuts[j], b = cuts[j + 1];
        int flags = (r == m - 1) ? kItemLast : 0;
        if (b - a > 0 && over(a, b)) flags |= kItemDirect;
        emit(T, l, a, b, flags);
      }
      ++T.num_steps;
    }
  }
}

}  // namespace

void build_items(DevGraph& d, const std::vector<int32_t>& lfo_ptr) {
  const HostLevels& h = d.host;
  const int G = d.grid;
  const auto& fp = h.fanin_ptr;
  // forward and batched forward: work = 1 + fanin arcs
  for (int pass = 0; pass < 2; ++pass) {
    const Caps caps = pass == 0 ? Caps{kFwdPins, kFwdArcs, 0} : Caps{kBFwdPins, kBFwdArcs, 0};
    cut_levels(
        pass == 0 ? d.fwd_items : d.bfwd_items, G, h.level_ptr, false,
        [&](int32_t p) { return int64_t(1) + (fp[p + 1] - fp[p]); },
        [&](int32_t a, int32_t b) { return b - a > caps.pins || fp[b] - fp[a] > caps.arcs; },
        [&](ItemTable& T, int l, int32_t a, int32_t b, int flags) {
          T.a.push_back(make_int4(a, b, fp[a], fp[b]));
          T.b.push_back(make_int4(l, flags, 0, 0));
        });
  }
  // backward: work = 1 + fanin arcs + light fanout entries, reverse level order
  cut_levels(
      d.bwd_items, G, h.level_ptr, true,
      [&](int32_t p) { return int64_t(1) + (fp[p + 1] - fp[p]) + (lfo_ptr[p + 1] - lfo_ptr[p]); },
      [&](int32_t a, int32_t b) {
        return b - a > kBwdPins || fp[b] - fp[a] > kBwdArcs || lfo_ptr[b] - lfo_ptr[a] > kBwdFanout;
      },
      [&](ItemTable& T, int l, int32_t a, int32_t b, int flags) {
        T.a.push_back(make_int4(a, b, lfo_ptr[a], lfo_ptr[b]));
        T.b.push_back(make_int4(fp[a], fp[b], l, flags));
      });
}

void build_fold_items(DevGraph& d, const FoldHost& f) {
  const int G = d.grid;
  const auto& hp = f.hd_ptr;
  // folded forward: work of a head = 1 + entries + folded entries
  cut_levels(
      d.fwdf_items, G, f.slevel_ptr, false,
      [&](int32_t h) { return int64_t(1) + (hp[h + 1] - hp[h]) + f.hd_nfold[h]; },
      [&](int32_t a, int32_t b) { return b - a > kFwdPins || hp[b] - hp[a] > kFwdArcs; },
      [&](ItemTable& T, int l, int32_t a, int32_t b, int flags) {
        T.a.push_back(make_int4(a, b, hp[a], hp[b]));
        T.b.push_back(make_int4(l, flags, 0, 0));
      });
  // folded batched forward (larger caps)
  cut_levels(
      d.bfwdf_items, G, f.slevel_ptr, false,
      [&](int32_t h) { return int64_t(1) + (hp[h + 1] - hp[h]) + f.hd_nfold[h]; },
      [&](int32_t a, int32_t b) { return b - a > kBFwdPins || hp[b] - hp[a] > kBFwdArcs; },
      [&](ItemTable& T, int l, int32_t a, int32_t b, int flags) {
        T.a.push_back(make_int4(a, b, hp[a], hp[b]));
        T.b.push_back(make_int4(l, flags, 0, 0));
      });
  // folded backward: reverse super-level order; work = 1 + entries + folded
  // entries + light fanout entries
  const auto& lp = f.hlfo_ptr;
  cut_levels(
      d.bwdf_items, G, f.slevel_ptr, true,
      [&](int32_t h) { return int64_t(1) + (hp[h + 1] - hp[h]) + f.hd_nfold[h] + (lp[h + 1] - lp[h]); },
      [&](int32_t a, int32_t b) {
        return b - a > kBwdPins || hp[b] - hp[a] > kBwdArcs || lp[b] - lp[a] > kBwdFanout;
      },
      [&](ItemTable& T, int l, int32_t a, int32_t b, int flags) {
        T.a.push_back(make_int4(a, b, lp[a], lp[b]));
        T.b.push_back(make_int4(hp[a], hp[b], l, flags));
      });
}

}  // namespace insta
