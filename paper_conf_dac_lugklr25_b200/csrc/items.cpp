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

}  // namespace

void build_items(DevGraph& d, const std::vector<int32_t>& lfo_ptr) {
  const HostLevels& h = d.host;
  const int G = d.grid;
  const int L = h.num_levels;
  for (int pass = 0; pass < 3; ++pass) {   // forward, backward, batched forward
    const bool bwd = pass == 1;
    ItemTable& T = pass == 0 ? d.fwd_items : (bwd ? d.bwd_items : d.bfwd_items);
    T = ItemTable();
    T.level_step0.assign(size_t(L), 0);
    T.level_steps.assign(size_t(L), 0);
    const Caps caps = bwd ? Caps{kBwdPins, kBwdArcs, kBwdFanout}
                          : (pass == 0 ? Caps{kFwdPins, kFwdArcs, 1 << 30} : Caps{kBFwdPins, kBFwdArcs, 1 << 30});
    std::vector<int64_t> prefix;
    std::vector<int32_t> cuts;
    for (int li = 0; li < L; ++li) {
      const int l = bwd ? (L - 1 - li) : li;
      const int32_t lo = h.level_ptr[l], hi = h.level_ptr[l + 1];
      prefix.assign(size_t(hi - lo) + 1, 0);
      for (int32_t p = lo; p < hi; ++p) {
        int64_t w = 1 + (h.fanin_ptr[p + 1] - h.fanin_ptr[p]);
        if (bwd) w += lfo_ptr[p + 1] - lfo_ptr[p];
        prefix[p - lo + 1] = prefix[p - lo] + w;
      }
      int64_t m = 1;
      for (;;) {
        quantile_cuts(prefix, lo, m * G, &cuts);
        bool ok = true;
        for (int64_t j = 0; j < m * G && ok; ++j) {
          const int32_t a = cuts[j], b = cuts[j + 1];
          if (b - a <= 1) continue;   // single pins are always accepted (direct if too big)
          const int64_t arcs = h.fanin_ptr[b] - h.fanin_ptr[a];
          const int64_t fo = bwd ? int64_t(lfo_ptr[b] - lfo_ptr[a]) : 0;
          if (b - a > caps.pins || arcs > caps.arcs || fo > caps.fanout) ok = false;
        }
        if (ok || m * G >= int64_t(hi - lo)) break;
        m *= 2;
      }
      // with m*G >= pins every chunk holds <= 1 pin, so the loop above terminates
      T.level_step0[l] = T.num_steps;
      T.level_steps[l] = int32_t(m);
      for (int64_t r = 0; r < m; ++r) {
        for (int c = 0; c < G; ++c) {
          const int64_t j = r * G + c;
          const int32_t a = cuts[j], b = cuts[j + 1];
          const int32_t alo = h.fanin_ptr[a], ahi = h.fanin_ptr[b];
          const int64_t arcs = ahi - alo;
          const int64_t fo = bwd ? int64_t(lfo_ptr[b] - lfo_ptr[a]) : 0;
          int flags = (r == m - 1) ? kItemLast : 0;
          if (b - a > caps.pins || arcs > caps.arcs || fo > caps.fanout) flags |= kItemDirect;
          if (!bwd) {
            T.a.push_back(make_int4(a, b, alo, ahi));
            T.b.push_back(make_int4(l, flags, 0, 0));
          } else {
            T.a.push_back(make_int4(a, b, lfo_ptr[a], lfo_ptr[b]));
            T.b.push_back(make_int4(alo, ahi, l, flags));
          }
        }
        ++T.num_steps;
      }
    }
  }
}

}  // namespace insta
