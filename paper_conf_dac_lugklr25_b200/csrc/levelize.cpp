// levelize.cpp -- host levelizer ("INSTA constructs and levelizes its
// timing graph for parallel arrival time propagation, where pins within the
// same level are processed independently ... topological sort").
//
// Frontier-synchronous Kahn: frontier 0 = indeg-0 pins; frontier l+1 = pins
// whose last unprocessed fanin was in frontier l.  A pin becomes ready exactly
// when its deepest source is processed, so frontier index = ASAP level =
// 1 + max level(source).  Each frontier is emitted sorted by caller pin id,
// which yields the canonical (level, id) order directly.  Fanin/fanout rows are
// filled by scanning arcs in ascending caller id, so rows come out sorted.
#include <algorithm>
#include <cstring>

#include "internal.h"

namespace insta {

insta_status levelize_host(int32_t n, int64_t e, const int32_t* from, const int32_t* to,
                           HostLevels* out, std::string* err) {
  if (n < 0 || n > kMaxPins || e < 0 || e >= (int64_t(1) << 31)) {
    *err = "levelize: size out of range (num_pins < 2^29, num_arcs < 2^31)";
    return INSTA_E_ARG;
  }
  if (e > 0 && (!from || !to)) { *err = "levelize: NULL arc arrays"; return INSTA_E_ARG; }
  for (int64_t a = 0; a < e; ++a) {
    if (uint32_t(from[a]) >= uint32_t(n) || uint32_t(to[a]) >= uint32_t(n)) {
      *err = "levelize: arc " + std::to_string(a) + " has a pin id out of range";
      return INSTA_E_ARG;
    }
  }
  HostLevels& h = *out;
  h = HostLevels();
  h.n = n;
  h.e = e;
  // out-adjacency by caller id (CSR over pins, targets only)
  std::vector<int32_t> optr(size_t(n) + 1, 0);
  std::vector<int32_t> oadj(static_cast<size_t>(e));
  std::vector<int32_t> remaining(size_t(n), 0);
  for (int64_t a = 0; a < e; ++a) { optr[from[a] + 1]++; remaining[to[a]]++; }
  for (int32_t p = 0; p < n; ++p) optr[p + 1] += optr[p];
  {
    std::vector<int32_t> cur(optr.begin(), optr.end() - 1);
    for (int64_t a = 0; a < e; ++a) oadj[cur[from[a]]++] = to[a];
  }
  h.level.assign(size_t(n), -1);
  h.order.clear();
  h.order.reserve(size_t(n));
  h.level_ptr.clear();
  std::vector<int32_t> frontier, next;
  for (int32_t p = 0; p < n; ++p)
    if (remaining[p] == 0) frontier.push_back(p);   // ascending already
  int32_t lvl = 0;
  while (!frontier.empty()) {
    h.level_ptr.push_back(int32_t(h.order.size()));
    next.clear();
    for (int32_t p : frontier) {
      h.level[p] = lvl;
      h.order.push_back(p);
      for (int32_t k = optr[p]; k < optr[p + 1]; ++k)
        if (--remaining[oadj[k]] == 0) next.push_back(oadj[k]);
    }
    std::sort(next.begin(), next.end());
    frontier.swap(next);
    ++lvl;
  }
  if (int64_t(h.order.size()) != n) {
    *err = "levelize: combinational loop (" + std::to_string(n - int64_t(h.order.size())) +
           " pins on or behind a cycle)";
    return INSTA_E_CYCLE;
  }
  h.level_ptr.push_back(n);
  h.num_levels = lvl;
  h.pos.assign(size_t(n), 0);
  for (int32_t k = 0; k < n; ++k) h.pos[h.order[k]] = k;

  h.fanin_ptr.assign(size_t(n) + 1, 0);
  h.fanout_ptr.assign(size_t(n) + 1, 0);
  for (int64_t a = 0; a < e; ++a) {
    h.fanin_ptr[h.pos[to[a]] + 1]++;
    h.fanout_ptr[h.pos[from[a]] + 1]++;
  }
  for (int32_t k = 0; k < n; ++k) {
    h.fanin_ptr[k + 1] += h.fanin_ptr[k];
    h.fanout_ptr[k + 1] += h.fanout_ptr[k];
  }
  h.fanin_arc.assign(size_t(e), 0);
  h.fanout_arc.assign(size_t(e), 0);
  std::vector<int32_t> ci(h.fanin_ptr.begin(), h.fanin_ptr.end() - 1);
  std::vector<int32_t> co(h.fanout_ptr.begin(), h.fanout_ptr.end() - 1);
  for (int64_t a = 0; a < e; ++a) {
    h.fanin_arc[ci[h.pos[to[a]]]++] = int32_t(a);
    h.fanout_arc[co[h.pos[from[a]]]++] = int32_t(a);
  }
  return INSTA_OK;
}

}  // namespace insta
