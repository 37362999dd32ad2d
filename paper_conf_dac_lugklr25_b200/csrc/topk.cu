// topk.cu -- Top-K statistical arrival propagation with unique startpoints and
// CPPR-aware endpoint slack (Alg 1 P:L70-73,
// Alg 2).
//
// Semantics.  Per pin and sink transition rf, a queue of K entries {mu, var,
// SP} descending in the corner arrival A = mu + N_sigma * sigma (Eq 1-3).  Alg
// 1 offers the candidates of a pin in the order (k outer, fanin arc inner, s
// innermost) to Alg 2, which keeps one entry per startpoint (replace only if
// strictly greater, re-bubble; insert only if strictly greater than the
// smallest).  That sequential procedure has a closed description: with t the
// position of a candidate in that order, the queue is the K largest
// startpoints ranked by the key (A desc, t asc) of each startpoint's best
// candidate (largest A, earliest t).  The kernel maintains exactly that set
// under an explicit (A, t) key, so it may consume candidates in any order and
// still reproduce the sequential result bit for bit, ties included (tested
// against the oracle's literal Alg 2 in dyadic mode).
//
// Execution.  One launch per level (the levels are wide and each (pin, rf)
// moves K entries per fanin arc, so a level is ~tens of us of HBM traffic and
// the launch latency is amortized).  A group of G = pow2(K) lanes owns one (pin,
// rf); lane k holds queue slot k in registers.  Per fanin arc and source
// transition, lane k loads the parent's slot k (16 B {mu, var} + 4 B SP,
// coalesced across the group), forms the candidate, and one ballot prunes
// every candidate whose key is below the queue's last slot (the common case
// once the queue is full).  Survivors are merged one at a time with ballots
// (startpoint match, insert position) and a one-lane shift (shfl_up).
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdint>
#include <vector>

#include "device_common.cuh"
#include "internal.h"

// resident blocks per SM the level kernel is compiled for (register budget)
#ifndef TK_MINB
#define TK_MINB 6
#endif

namespace insta {

#ifdef TK_STATS
__device__ unsigned long long tk_stats[33];   // merge batches by survivor count (debug builds)
#endif

struct TkParams {
  int32_t lo, hi, K;
  const int32_t* __restrict__ list;   // canonical pins of this launch: list[lo..hi)
  double ns;
  const int32_t* __restrict__ fanin_ptr;
  const int32_t* __restrict__ fin_src;
  const float4* __restrict__ fin_ms;
  double2* q;     // [n][2][K] {mu, var}
  int32_t* qsp;   // [n][2][K] canonical startpoint, -1 = empty
};

// (A, t) key order: larger A first, earlier candidate first among equal A
__device__ __forceinline__ bool key_gt(double a, int ta, double b, int tb) {
  return a > b || (a == b && ta < tb);
}

// startpoints: entry 0 = the clock arrival, SP = the pin itself
__global__ void tk_src_kernel(int n_src, int K, const float4* __restrict__ src_ms, double2* q, int32_t* qsp) {
  const long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (x >= 2LL * n_src * K) return;
  const int k = int(x % K), rf = int((x / K) & 1), p = int(x / (2LL * K));
  if (k == 0) {
    const float4 v = __ldg(src_ms + p);
    const double s = double(rf ? v.w : v.z);
    q[x] = make_double2(double(rf ? v.y : v.x), s * s);
    qsp[x] = p;
  } else {
    q[x] = make_double2(0.0, 0.0);
    qsp[x] = -1;
  }
}

// A queue slot or a candidate: corner arrival A, key position t, distribution, startpoint.
struct TkEnt {
  double A, mu, var;
  int t, sp;
};

__device__ __forceinline__ TkEnt tk_empty() { return TkEnt{-INFINITY, 0.0, 0.0, INT_MAX, -1}; }

__device__ __forceinline__ TkEnt shfl_ent(unsigned gm, const TkEnt& e, int src) {
  TkEnt o;
  o.A = __shfl_sync(gm, e.A, src);
  o.mu = __shfl_sync(gm, e.mu, src);
  o.var = __shfl_sync(gm, e.var, src);
  o.t = __shfl_sync(gm, e.t, src);
  o.sp = __shfl_sync(gm, e.sp, src);
  return o;
}

template <int G>
struct Log2 {
  static constexpr int v = G <= 1 ? 0 : 1 + Log2<(G > 1 ? G / 2 : 1)>::v;
};
template <>
struct Log2<1> {
  static constexpr int v = 0;
};

// Bitonic sort of (A, t) keys over the G lanes of a group, descending; idx
// follows its key (the lane that held it before the sort).
template <int G>
__device__ __forceinline__ void bitonic_desc(unsigned gm, int gl, double& sA, int& st, int& idx) {
#pragma unroll
  for (int k = 2; k <= G; k <<= 1) {
#pragma unroll
    for (int jj = k >> 1; jj > 0; jj >>= 1) {
      const double oA = __shfl_xor_sync(gm, sA, jj, G);
      const int ot = __shfl_xor_sync(gm, st, jj, G), oi = __shfl_xor_sync(gm, idx, jj, G);
      const bool want_max = ((gl & jj) == 0) == ((gl & k) == 0);
      if (want_max ? key_gt(oA, ot, sA, st) : key_gt(sA, st, oA, ot)) {
        sA = oA;
        st = ot;
        idx = oi;
      }
    }
  }
}

// parent slot loads of one batch (fanin arc held by lane `src`, source
// transition index si); the {mu, var} load does not wait for the startpoint
// word (empty slots hold zeros)
__device__ __forceinline__ void tk_issue(const TkParams& P, unsigned gm, int src, int32_t wl, int rf, int si, int K,
                                         int gl, bool slot, int& csp, double2& pv) {
  const int32_t w = __shfl_sync(gm, wl, src);
  const size_t ps = (size_t(w & kSrcMask) * 2 + src_tr(rf, int(uint32_t(w) >> kUnateShift), si)) * K + gl;
  csp = slot ? __ldg(P.qsp + ps) : -1;
  pv = slot ? __ldg(P.q + ps) : make_double2(0.0, 0.0);
}

template <int G>
__global__ void __launch_bounds__(256, TK_MINB) tk_level_kernel(TkParams P) {
  // per-group scatter area of the bulk merge (one slot per thread of the block)
  __shared__ double smA[256], smMu[256], smVar[256];
  __shared__ int smT[256], smSp[256];
  const int lane = threadIdx.x & 31;
  const int gl = lane & (G - 1), gbase = lane & ~(G - 1), tbase = threadIdx.x & ~(G - 1);
  const unsigned gm = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
  const long long grp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) / G;
  if (grp >= 2LL * (P.hi - P.lo)) return;   // uniform within a group
  const int i = __ldg(P.list + P.lo + int(grp >> 1)), rf = int(grp & 1), K = P.K;
  const bool slot = gl < K;
  const int last = gbase + K - 1;
  TkEnt q = tk_empty();
  bool first = true;
  const int b0 = __ldg(P.fanin_ptr + i), b1 = __ldg(P.fanin_ptr + i + 1), nf = b1 - b0;
  for (int c0 = b0; c0 < b1; c0 += G) {
    // the row's topology, one fanin arc per lane (rows longer than G in chunks)
    const int cn = min(G, b1 - c0);
    int32_t wl = 0;
    float4 msl = make_float4(0.f, 0.f, 0.f, 0.f);
    if (gl < cn) {
      wl = __ldg(P.fin_src + c0 + gl);
      msl = __ldg(P.fin_ms + c0 + gl);
    }
    // parent slot loads run one batch ahead of the merge; the {mu, var} load
    // does not wait for the startpoint word (empty slots hold zeros)
    int csp_n;
    double2 pv_n;
    tk_issue(P, gm, gbase + 0, wl, rf, 0, K, gl, slot, csp_n, pv_n);
    for (int x = 0; x < cn; ++x) {
      const int32_t w = __shfl_sync(gm, wl, gbase + x);
      const int u = int(uint32_t(w) >> kUnateShift);
      const float am_f = __shfl_sync(gm, rf ? msl.y : msl.x, gbase + x);
      const float se_f = __shfl_sync(gm, rf ? msl.w : msl.z, gbase + x);
      const double am = double(am_f), se = double(se_f);
      for (int si = 0; si < n_src_tr(u); ++si) {
        const int csp = csp_n;
        const double2 pv = pv_n;
        {
          int nx = x, nsi = si + 1;
          if (nsi >= n_src_tr(u)) {
            nx = x + 1;
            nsi = 0;
          }
          if (nx < cn) tk_issue(P, gm, gbase + nx, wl, rf, nsi, K, gl, slot, csp_n, pv_n);
        }
        TkEnt c;
        c.sp = csp;
        c.t = (gl * nf + (c0 + x - b0)) * 2 + si;   // Alg 1 order: k outer, arcs, s
        c.mu = pv.x + am;                            // Eq 1 (l.12)
        c.var = pv.y + se * se;                      // Eq 2 (l.13)
        c.A = csp >= 0 ? c.mu + P.ns * double(sigma_of(c.var)) : -INFINITY;   // Eq 3 (l.14)
        if (first) {
          // first batch into an empty queue: one parent's queue has unique
          // startpoints, so Alg 2 reduces to ordering the candidates by key
          first = false;
          const double nA = __shfl_down_sync(gm, c.A, 1, G);
          const int nt = __shfl_down_sync(gm, c.t, 1, G);
          int idx = gl;
          if (__ballot_sync(gm, gl + 1 < G && key_gt(nA, nt, c.A, c.t)) & gm) {
            double sA = c.A;
            int st = csp >= 0 ? c.t : INT_MAX;
            bitonic_desc<G>(gm, gl, sA, st, idx);
          }
          q = shfl_ent(gm, c, gbase + idx);
          if (q.sp < 0) q = tk_empty();
          continue;
        }
        // one ballot prunes every candidate below the queue's last slot: it can
        // neither enter nor beat its startpoint's entry
        const double mA = __shfl_sync(gm, q.A, last);
        const int mt = __shfl_sync(gm, q.t, last);
        const bool surv = csp >= 0 && key_gt(c.A, c.t, mA, mt);
        unsigned m = __ballot_sync(gm, surv) & gm;
#ifdef TK_STATS
        if (gl == 0) atomicAdd(&tk_stats[min(__popc(m), 32)], 1ull);
#endif
        if (__popc(m) <= 2) {
          while (m) {   // Alg 2, one survivor at a time
            const int src = __ffs(m) - 1;
            m &= m - 1;
            const TkEnt n = shfl_ent(gm, c, src);
            const unsigned fm = __ballot_sync(gm, slot && q.sp == n.sp) & gm;
            int f;
            if (fm) {                                      // Step 1: the startpoint is queued
              f = __ffs(fm) - 1;
              if (!key_gt(n.A, n.t, __shfl_sync(gm, q.A, f), __shfl_sync(gm, q.t, f))) continue;
              f -= gbase;
            } else {                                       // Step 2: a new startpoint
              if (!key_gt(n.A, n.t, __shfl_sync(gm, q.A, last), __shfl_sync(gm, q.t, last))) continue;
              f = K - 1;                                   // the last entry falls off
            }
            const int p = __popc(__ballot_sync(gm, slot && key_gt(q.A, q.t, n.A, n.t)) & gm);
            TkEnt up;
            up.A = __shfl_up_sync(gm, q.A, 1, G);
            up.mu = __shfl_up_sync(gm, q.mu, 1, G);
            up.var = __shfl_up_sync(gm, q.var, 1, G);
            up.t = __shfl_up_sync(gm, q.t, 1, G);
            up.sp = __shfl_up_sync(gm, q.sp, 1, G);
            if (gl > p && gl <= f) q = up;
            else if (gl == p) q = n;
          }
          continue;
        }
        // bulk merge of many survivors: (1) match each survivor's startpoint
        // in the queue; a matched one replaces its entry only if its key is
        // larger, else it is dropped; (2) sort the kept candidates; (3) rank
        // every alive queue entry and kept candidate in the union by binary
        // search in the other sorted list; (4) scatter the top K through
        // shared memory.
        int f = -1;
        const int ssp = surv ? csp : -1;
        if (G >= 4) {
          // __match_any over half-groups: lanes [0, H) carry queue slots,
          // lanes [H, G) survivors' startpoints; four calls cover all pairs
          constexpr int H = G / 2;
#pragma unroll
          for (int qh = 0; qh < 2; ++qh) {
#pragma unroll
            for (int ch = 0; ch < 2; ++ch) {
              const int qs = __shfl_sync(gm, q.sp, gbase + qh * H + (gl & (H - 1)));
              const int cs = __shfl_sync(gm, ssp, gbase + ch * H + (gl & (H - 1)));
              const unsigned v = gl < H ? (qs >= 0 ? unsigned(qs) : 0x40000000u | gl)
                                        : (cs >= 0 ? unsigned(cs) : 0x60000000u | gl);
              const unsigned qb = (__match_any_sync(gm, v) >> gbase) & ((1u << H) - 1u);
              const int fq = qb ? qh * H + __ffs(qb) - 1 : -1;
              const int r = __shfl_sync(gm, fq, gbase + H + (gl & (H - 1)));
              if ((gl >> Log2<H>::v) == ch && r >= 0) f = r;
            }
          }
        } else {
          for (int r = 0; r < K; ++r)
            if (__shfl_sync(gm, q.sp, gbase + r) == ssp && ssp >= 0) f = r;
        }
        const double fA = __shfl_sync(gm, q.A, gbase + max(f, 0));
        const int ft = __shfl_sync(gm, q.t, gbase + max(f, 0));
        bool keep = surv;
        unsigned deadbit = 0u;
        if (surv && f >= 0) {
          if (key_gt(c.A, c.t, fA, ft)) deadbit = 1u << f;
          else keep = false;
        }
        const unsigned dead = __reduce_or_sync(gm, deadbit);
        // kept candidates compacted in lane order (a parent's queue order is
        // mostly preserved by Eq 1-3), then sorted only if out of order
        const unsigned km = (__ballot_sync(gm, keep) & gm) >> gbase;
        const int nC = __popc(km);
        int idx = gl < nC ? int(__fns(km, 0, gl + 1)) : gl;
        double sA = __shfl_sync(gm, c.A, gbase + idx);
        int st = __shfl_sync(gm, c.t, gbase + idx);
        if (gl >= nC) {
          sA = -INFINITY;
          st = INT_MAX;
        }
        {
          const double nA = __shfl_down_sync(gm, sA, 1, G);
          const int nt = __shfl_down_sync(gm, st, 1, G);
          if (__ballot_sync(gm, gl + 1 < nC && key_gt(nA, nt, sA, st)) & gm) bitonic_desc<G>(gm, gl, sA, st, idx);
        }
        const unsigned qv = (__ballot_sync(gm, slot && q.sp >= 0) & gm) >> gbase;
        const int nQ = __popc(qv);
        int lo = 0, hi = nC;   // kept candidates ahead of my queue entry
#pragma unroll
        for (int it = 0; it <= Log2<G>::v; ++it) {
          const int mid = (lo + hi) >> 1;
          const double xA = __shfl_sync(gm, sA, gbase + min(mid, G - 1));
          const int xt = __shfl_sync(gm, st, gbase + min(mid, G - 1));
          if (lo < hi) {
            if (key_gt(xA, xt, q.A, q.t)) lo = mid + 1;
            else hi = mid;
          }
        }
        const int rankQ = __popc(qv & ~dead & ((1u << gl) - 1u)) + lo;
        int lo2 = 0, hi2 = nQ;   // queue entries ahead of my sorted candidate
#pragma unroll
        for (int it = 0; it <= Log2<G>::v; ++it) {
          const int mid = (lo2 + hi2) >> 1;
          const double xA = __shfl_sync(gm, q.A, gbase + min(mid, G - 1));
          const int xt = __shfl_sync(gm, q.t, gbase + min(mid, G - 1));
          if (lo2 < hi2) {
            if (key_gt(xA, xt, sA, st)) lo2 = mid + 1;
            else hi2 = mid;
          }
        }
        const int rankC = gl + lo2 - __popc(lo2 >= 32 ? dead : dead & ((1u << lo2) - 1u));
        const TkEnt gc = shfl_ent(gm, c, gbase + idx);
        __syncwarp(gm);
        if (slot && q.sp >= 0 && !((dead >> gl) & 1u) && rankQ < K) {
          smA[tbase + rankQ] = q.A;
          smMu[tbase + rankQ] = q.mu;
          smVar[tbase + rankQ] = q.var;
          smT[tbase + rankQ] = q.t;
          smSp[tbase + rankQ] = q.sp;
        }
        if (gl < nC && rankC < K) {
          smA[tbase + rankC] = gc.A;
          smMu[tbase + rankC] = gc.mu;
          smVar[tbase + rankC] = gc.var;
          smT[tbase + rankC] = gc.t;
          smSp[tbase + rankC] = gc.sp;
        }
        __syncwarp(gm);
        if (gl < min(K, nQ - __popc(dead) + nC)) {
          q.A = smA[tbase + gl];
          q.mu = smMu[tbase + gl];
          q.var = smVar[tbase + gl];
          q.t = smT[tbase + gl];
          q.sp = smSp[tbase + gl];
        } else {
          q = tk_empty();
        }
        __syncwarp(gm);
      }
    }
  }
  if (slot) {
    const size_t o = (size_t(i) * 2 + rf) * K + gl;
    P.q[o] = make_double2(q.mu, q.var);
    P.qsp[o] = q.sp;
  }
}

// Pins with exactly one fanin arc that is not non-unate (net sinks, the
// inputs of one-input cells): one batch from one parent, whose startpoints
// are unique, so Alg 2 reduces to ordering the K candidates by key.  A lean
// kernel (no merge state) that runs at full occupancy.
template <int G>
__global__ void __launch_bounds__(256, 8) tk_one_kernel(TkParams P) {
  const int lane = threadIdx.x & 31;
  const int gl = lane & (G - 1), gbase = lane & ~(G - 1);
  const unsigned gm = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
  const long long grp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) / G;
  if (grp >= 2LL * (P.hi - P.lo)) return;
  const int i = __ldg(P.list + P.lo + int(grp >> 1)), rf = int(grp & 1), K = P.K;
  const bool slot = gl < K;
  const int a = __ldg(P.fanin_ptr + i);
  const int32_t w = __ldg(P.fin_src + a);
  const float4 ms = __ldg(P.fin_ms + a);
  const size_t ps = (size_t(w & kSrcMask) * 2 + src_tr(rf, int(uint32_t(w) >> kUnateShift), 0)) * K + gl;
  const int csp = slot ? __ldg(P.qsp + ps) : -1;
  const double2 pv = slot ? __ldg(P.q + ps) : make_double2(0.0, 0.0);
  const double se = double(rf ? ms.w : ms.z);
  const double mu = pv.x + double(rf ? ms.y : ms.x);   // Eq 1
  const double var = pv.y + se * se;                   // Eq 2
  double A = csp >= 0 ? mu + P.ns * double(sigma_of(var)) : -INFINITY;   // Eq 3
  int t = csp >= 0 ? gl * 2 : INT_MAX;                 // single arc: t = 2k
  const double nA = __shfl_down_sync(gm, A, 1, G);
  const int nt = __shfl_down_sync(gm, t, 1, G);
  int idx = gl;
  if (__ballot_sync(gm, gl + 1 < G && key_gt(nA, nt, A, t)) & gm) bitonic_desc<G>(gm, gl, A, t, idx);
  const double omu = __shfl_sync(gm, mu, gbase + idx), ovar = __shfl_sync(gm, var, gbase + idx);
  const int osp = __shfl_sync(gm, csp, gbase + idx);
  if (slot) {
    const size_t o = (size_t(i) * 2 + rf) * K + gl;
    P.q[o] = osp >= 0 ? make_double2(omu, ovar) : make_double2(0.0, 0.0);
    P.qsp[o] = osp;
  }
}

// K in (32, kTkWideMax]: a warp per (pin, rf) with its queue in shared memory
// (kTkWideCap entries: the K queue slots plus one chunk of new candidates,
// padded to a power of two).  Candidates arrive 32 at a time (one parent
// queue's slots, unique startpoints, in Alg 1's k order); when the queue is
// full, those whose (A, t) key is below its last slot are pruned (they can
// neither enter nor beat their startpoint's entry); each survivor looks up its
// startpoint in the queue (a found one replaces its entry only with a larger
// key, else it is dropped), new ones are appended, and the queue is re-sorted
// by key (warp bitonic sort in shared memory) and cut to K.  This maintains
// the R19 closed form (the K best startpoints by their best candidate's key),
// so the result equals the literal sequential Alg 2 bit for bit.
constexpr int kTkWideMax = 128, kTkWideCap = 256, kTkWideWarps = 4;
struct TkWideSm {
  double A[kTkWideCap], mu[kTkWideCap], var[kTkWideCap];
  int t[kTkWideCap], sp[kTkWideCap];
};

__device__ __forceinline__ void tk_sm_put(TkWideSm& Q, int j, const TkEnt& c) {
  Q.A[j] = c.A;
  Q.mu[j] = c.mu;
  Q.var[j] = c.var;
  Q.t[j] = c.t;
  Q.sp[j] = c.sp;
}

__device__ __forceinline__ void tk_sm_swap(TkWideSm& Q, int i, int j) {
  const double a = Q.A[i], m = Q.mu[i], v = Q.var[i];
  const int t = Q.t[i], sp = Q.sp[i];
  Q.A[i] = Q.A[j];
  Q.mu[i] = Q.mu[j];
  Q.var[i] = Q.var[j];
  Q.t[i] = Q.t[j];
  Q.sp[i] = Q.sp[j];
  Q.A[j] = a;
  Q.mu[j] = m;
  Q.var[j] = v;
  Q.t[j] = t;
  Q.sp[j] = sp;
}

// descending (A, t) order of Q[0, n): bitonic over the next power of two, the tail padded empty
__device__ __forceinline__ void tk_sm_sort(TkWideSm& Q, int n, int lane) {
  int P2 = 1;
  while (P2 < n) P2 <<= 1;
  for (int j = n + lane; j < P2; j += 32) tk_sm_put(Q, j, tk_empty());
  __syncwarp();
  for (int size = 2; size <= P2; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int p = lane; p < (P2 >> 1); p += 32) {
        const int i = 2 * p - (p & (stride - 1)), j = i + stride;
        const bool desc = (i & size) == 0;
        const bool sw = desc ? key_gt(Q.A[j], Q.t[j], Q.A[i], Q.t[i]) : key_gt(Q.A[i], Q.t[i], Q.A[j], Q.t[j]);
        if (sw) tk_sm_swap(Q, i, j);
      }
      __syncwarp();
    }
  }
}

__global__ void __launch_bounds__(32 * kTkWideWarps) tk_wide_kernel(TkParams P) {
  __shared__ TkWideSm S[kTkWideWarps];
  const int lane = threadIdx.x & 31;
  TkWideSm& Q = S[threadIdx.x >> 5];
  const long long grp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  if (grp >= 2LL * (P.hi - P.lo)) return;   // uniform within the warp
  const int i = __ldg(P.list + P.lo + int(grp >> 1)), rf = int(grp & 1), K = P.K;
  const int b0 = __ldg(P.fanin_ptr + i), b1 = __ldg(P.fanin_ptr + i + 1), nf = b1 - b0;
  int n = 0;
  for (int r = b0; r < b1; ++r) {   // fanin arcs in row order (Alg 1 l.7-8)
    const int32_t w = __ldg(P.fin_src + r);
    const int u = int(uint32_t(w) >> kUnateShift);
    const float4 ms = __ldg(P.fin_ms + r);
    const double am = double(rf ? ms.y : ms.x), se = double(rf ? ms.w : ms.z);
    for (int si = 0; si < n_src_tr(u); ++si) {
      const size_t ps0 = (size_t(w & kSrcMask) * 2 + src_tr(rf, u, si)) * K;
      for (int k0 = 0; k0 < K; k0 += 32) {
        const int k = k0 + lane;
        const int csp = k < K ? __ldg(P.qsp + ps0 + k) : -1;
        const double2 pv = k < K ? __ldg(P.q + ps0 + k) : make_double2(0.0, 0.0);
        TkEnt c;
        c.sp = csp;
        c.t = (k * nf + (r - b0)) * 2 + si;          // Alg 1 order: k outer, arcs, s
        c.mu = pv.x + am;                            // Eq 1 (l.12)
        c.var = pv.y + se * se;                      // Eq 2 (l.13)
        c.A = csp >= 0 ? c.mu + P.ns * double(sigma_of(c.var)) : -INFINITY;   // Eq 3 (l.14)
        bool live = csp >= 0;
        if (n == K) live = live && key_gt(c.A, c.t, Q.A[K - 1], Q.t[K - 1]);
        if (!__ballot_sync(0xffffffffu, live)) continue;
        int f = -1;
        if (live)
          for (int j = 0; j < n; ++j)
            if (Q.sp[j] == csp) {
              f = j;
              break;
            }
        const bool rep = live && f >= 0 && key_gt(c.A, c.t, Q.A[f], Q.t[f]);
        const bool ins = live && f < 0;
        __syncwarp();
        if (rep) tk_sm_put(Q, f, c);
        const unsigned mi = __ballot_sync(0xffffffffu, ins);
        if (ins) tk_sm_put(Q, n + __popc(mi & ((1u << lane) - 1u)), c);
        const bool changed = __ballot_sync(0xffffffffu, rep || ins) != 0u;
        __syncwarp();
        if (!changed) continue;
        const int n2 = n + __popc(mi);
        tk_sm_sort(Q, n2, lane);
        n = min(n2, K);
      }
    }
  }
  for (int k = lane; k < K; k += 32) {
    const size_t o = (size_t(i) * 2 + rf) * K + k;
    const bool v = k < n;
    P.q[o] = v ? make_double2(Q.mu[k], Q.var[k]) : make_double2(0.0, 0.0);
    P.qsp[o] = v ? Q.sp[k] : -1;
  }
}

// Single-arc pins at K > 32 (a unate fanin arc: 11.2M of 15M pins at C4): the queue is the
// parent's, each slot shifted by the arc (Eq 1-3) -- one parent's startpoints are unique, so
// (R19) only the order by key (A desc, t = 2k asc) can change.  A warp per (pin, rf), K / 32
// slots per lane; the usual case (already in key order, one ballot over adjacent pairs) is
// written straight back, otherwise the warp sorts in shared memory (tk_sm_sort) -- the same
// queue the merging kernel builds for one arc, bit for bit.
__global__ void __launch_bounds__(32 * kTkWideWarps) tk_one_wide_kernel(TkParams P) {
  __shared__ TkWideSm S[kTkWideWarps];
  const int lane = threadIdx.x & 31;
  TkWideSm& Q = S[threadIdx.x >> 5];
  const long long grp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  if (grp >= 2LL * (P.hi - P.lo)) return;   // uniform within the warp
  const int i = __ldg(P.list + P.lo + int(grp >> 1)), rf = int(grp & 1), K = P.K;
  const int a = __ldg(P.fanin_ptr + i);
  const int32_t w = __ldg(P.fin_src + a);
  const float4 ms = __ldg(P.fin_ms + a);
  const size_t ps = (size_t(w & kSrcMask) * 2 + src_tr(rf, int(uint32_t(w) >> kUnateShift), 0)) * K;
  const double am = double(rf ? ms.y : ms.x), se = double(rf ? ms.w : ms.z);
  constexpr int kPer = kTkWideMax / 32;
  TkEnt c[kPer];
#pragma unroll
  for (int j = 0; j < kPer; ++j) {
    const int k = 32 * j + lane;
    const int csp = k < K ? __ldg(P.qsp + ps + k) : -1;
    const double2 pv = k < K ? __ldg(P.q + ps + k) : make_double2(0.0, 0.0);
    c[j].sp = csp;
    c[j].mu = pv.x + am;                                 // Eq 1
    c[j].var = pv.y + se * se;                           // Eq 2
    c[j].A = csp >= 0 ? c[j].mu + P.ns * double(sigma_of(c[j].var)) : -INFINITY;   // Eq 3
    c[j].t = csp >= 0 ? 2 * k : INT_MAX;                 // single arc: t = 2k
  }
  // in key order already?  pairs (k, k + 1) within a row of 32 and across rows
  bool bad = false;
#pragma unroll
  for (int j = 0; j < kPer; ++j) {
    const double nA = __shfl_down_sync(0xffffffffu, c[j].A, 1);
    const int nt = __shfl_down_sync(0xffffffffu, c[j].t, 1);
    const double xA = j + 1 < kPer ? __shfl_sync(0xffffffffu, c[j + 1 < kPer ? j + 1 : j].A, 0) : -INFINITY;
    const int xt = j + 1 < kPer ? __shfl_sync(0xffffffffu, c[j + 1 < kPer ? j + 1 : j].t, 0) : INT_MAX;
    const int k = 32 * j + lane;
    if (lane < 31 && k + 1 < K) bad |= key_gt(nA, nt, c[j].A, c[j].t);
    if (lane == 31 && k + 1 < K && j + 1 < kPer) bad |= key_gt(xA, xt, c[j].A, c[j].t);
  }
  if (__ballot_sync(0xffffffffu, bad)) {   // reorder by key in shared memory
#pragma unroll
    for (int j = 0; j < kPer; ++j)
      if (32 * j + lane < K) tk_sm_put(Q, 32 * j + lane, c[j]);
    __syncwarp();
    tk_sm_sort(Q, K, lane);
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
      const int k = 32 * j + lane;
      if (k < K) {
        c[j].A = Q.A[k];
        c[j].mu = Q.mu[k];
        c[j].var = Q.var[k];
        c[j].t = Q.t[k];
        c[j].sp = Q.sp[k];
      }
    }
  }
#pragma unroll
  for (int j = 0; j < kPer; ++j) {
    const int k = 32 * j + lane;
    if (k < K) {
      const size_t o = (size_t(i) * 2 + rf) * K + k;
      P.q[o] = c[j].sp >= 0 ? make_double2(c[j].mu, c[j].var) : make_double2(0.0, 0.0);
      P.qsp[o] = c[j].sp;
    }
  }
}

// CPPR slack: warp per endpoint; slack = min over (rf, k) of
// RAT(ep, SP_k)[rf] - A_k[rf], the first minimum in (rf, k) order wins.
__global__ void __launch_bounds__(256)
tk_slack_kernel(int num_ep, int K, double ns, const int32_t* __restrict__ ep_pin, const float2* __restrict__ ep_rat,
                const int32_t* __restrict__ rat_ptr, const int32_t* __restrict__ rat_sp,
                const float2* __restrict__ rat_val, const double2* __restrict__ q, const int32_t* __restrict__ qsp,
                double* slack, int32_t* star) {
  const int ep = int((blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5), lane = threadIdx.x & 31;
  if (ep >= num_ep) return;
  const int p = __ldg(ep_pin + ep);
  const float2 dr = __ldg(ep_rat + ep);
  const int r0 = rat_ptr ? __ldg(rat_ptr + ep) : 0, r1 = rat_ptr ? __ldg(rat_ptr + ep + 1) : 0;
  double best = INFINITY;
  int bidx = INT_MAX;
  for (int x = lane; x < 2 * K; x += 32) {
    const int rf = x / K;
    const size_t o = size_t(p) * 2 * K + x;
    const int sp = __ldg(qsp + o);
    if (sp < 0) continue;
    const double2 v = __ldg(q + o);
    const double A = v.x + ns * double(sigma_of(v.y));
    float rat = rf ? dr.y : dr.x;
    int lo = r0, hi = r1;   // rows are sorted by canonical startpoint
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (__ldg(rat_sp + mid) < sp) lo = mid + 1;
      else hi = mid;
    }
    if (lo < r1 && __ldg(rat_sp + lo) == sp) {
      const float2 rv = __ldg(rat_val + lo);
      rat = rf ? rv.y : rv.x;
    }
    const double s = double(rat) - A;
    if (s < best) {   // x increases per lane: strict keeps the first
      best = s;
      bidx = x;
    }
  }
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) {
    const double ob = __shfl_xor_sync(0xffffffffu, best, d);
    const int oi = __shfl_xor_sync(0xffffffffu, bidx, d);
    if (ob < best || (ob == best && oi < bidx)) {
      best = ob;
      bidx = oi;
    }
  }
  if (lane == 0) {
    slack[ep] = best;
    star[ep] = bidx == INT_MAX ? -1 : __ldg(qsp + size_t(p) * 2 * K + bidx) | ((bidx / K) << 30);
    star[num_ep + ep] = bidx == INT_MAX ? -1 : bidx % K;
  }
}

// WNS / TNS / violations in a fixed order (one block): contiguous chunks per
// thread summed in endpoint order, then a fixed tree.
__global__ void __launch_bounds__(1024) tk_reduce_kernel(int num_ep, const double* __restrict__ slack, double* out) {
  __shared__ double s_t[1024], s_w[1024], s_n[1024];
  const int t = threadIdx.x;
  const int ch = (num_ep + 1023) / 1024;
  double tns = 0.0, wns = 0.0, nv = 0.0;
  for (int e = t * ch; e < min(num_ep, (t + 1) * ch); ++e) {
    const double s = slack[e];
    if (s < 0.0) {
      tns += s;
      nv += 1.0;
    }
    wns = fmin(wns, s);
  }
  s_t[t] = tns;
  s_w[t] = wns;
  s_n[t] = nv;
  __syncthreads();
  for (int d = 512; d > 0; d >>= 1) {
    if (t < d) {
      s_t[t] += s_t[t + d];
      s_w[t] = fmin(s_w[t], s_w[t + d]);
      s_n[t] += s_n[t + d];
    }
    __syncthreads();
  }
  if (t == 0) {
    out[0] = s_w[0];
    out[1] = s_t[0];
    out[2] = s_n[0];
  }
}

// caller-order export of the queues (and of the per-endpoint slack / critical startpoint)
__global__ void tk_export_kernel(int n, int K, double ns, const int32_t* __restrict__ order, const double2* __restrict__ q,
                                 const int32_t* __restrict__ qsp, float* A, float* mean, float* sigma, int32_t* sp) {
  const long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (x >= 2LL * n * K) return;
  const int p = int(x / (2LL * K));
  const size_t o = size_t(__ldg(order + p)) * 2 * K + size_t(x % (2LL * K));
  const int s = __ldg(qsp + x);
  const double2 v = __ldg(q + x);
  const float sg = sigma_of(v.y);
  if (A) A[o] = s >= 0 ? float(v.x + ns * double(sg)) : -INFINITY;
  if (mean) mean[o] = s >= 0 ? float(v.x) : 0.f;
  if (sigma) sigma[o] = s >= 0 ? sg : 0.f;
  if (sp) sp[o] = s >= 0 ? __ldg(order + s) : -1;
}

__global__ void tk_export_slack_kernel(int num_ep, const int32_t* __restrict__ order, const double* __restrict__ slack,
                                       const int32_t* __restrict__ star, float* out, int32_t* sp_star, uint8_t* rf_star,
                                       int32_t* k_star) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= num_ep) return;
  const int32_t w = star[e];
  if (out) out[e] = float(slack[e]);
  if (sp_star) sp_star[e] = w < 0 ? -1 : __ldg(order + (w & ((1 << 30) - 1)));
  if (rf_star) rf_star[e] = w < 0 ? 0 : uint8_t(uint32_t(w) >> 30);
  if (k_star) k_star[e] = star[num_ep + e];
}

// --------------------------------------------------------------------------
// host launchers
// --------------------------------------------------------------------------
static int pow2_group(int K) {
  int G = 1;
  while (G < K) G <<= 1;
  return G;
}

int ensure_topk(DevGraph& g, int K) {
  if (!g.tk_list && g.n > 0) {
    // per level: single-arc (not non-unate) pins first, then the merging ones
    std::vector<int32_t> fsrc(size_t(std::max<int64_t>(g.e, 1)));
    if (g.e > 0) {
      cudaError_t e = cudaMemcpy(fsrc.data(), g.fin_src, sizeof(int32_t) * size_t(g.e), cudaMemcpyDeviceToHost);
      if (e != cudaSuccess) return int(e);
    }
    const std::vector<int32_t>& lp = g.host.level_ptr;
    const std::vector<int32_t>& fp = g.host.fanin_ptr;
    std::vector<int32_t> list;
    list.reserve(size_t(g.n));
    g.tk_one_ptr.assign(size_t(g.num_levels) + 1, 0);
    g.tk_multi_ptr.assign(size_t(g.num_levels) + 1, 0);
    for (int l = 0; l < g.num_levels; ++l) {
      g.tk_one_ptr[l] = int32_t(list.size());
      if (l > 0)
        for (int p = lp[l]; p < lp[l + 1]; ++p)
          if (fp[p + 1] - fp[p] == 1 && (uint32_t(fsrc[fp[p]]) >> kUnateShift) != 2u) list.push_back(p);
      g.tk_multi_ptr[l] = int32_t(list.size());
      if (l > 0)
        for (int p = lp[l]; p < lp[l + 1]; ++p)
          if (!(fp[p + 1] - fp[p] == 1 && (uint32_t(fsrc[fp[p]]) >> kUnateShift) != 2u)) list.push_back(p);
    }
    g.tk_one_ptr[g.num_levels] = g.tk_multi_ptr[g.num_levels] = int32_t(list.size());
    cudaError_t e = cudaMalloc(&g.tk_list, sizeof(int32_t) * std::max<size_t>(list.size(), 1));
    if (e == cudaSuccess && !list.empty())
      e = cudaMemcpy(g.tk_list, list.data(), sizeof(int32_t) * list.size(), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return int(e);
  }
  if (!g.tk_side) {
    cudaStream_t s2;
    cudaError_t e = cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    if (e != cudaSuccess) return int(e);
    g.tk_side = s2;
    cudaEvent_t* ev = reinterpret_cast<cudaEvent_t*>(g.tk_ev);
    for (int k = 0; k < 2 && e == cudaSuccess; ++k) e = cudaEventCreateWithFlags(&ev[k], cudaEventDisableTiming);
    if (e != cudaSuccess) return int(e);
  }
  if (g.tk_K == K && g.tk_q) return 0;
  if (g.tk_q) cudaFree(g.tk_q);
  if (g.tk_sp) cudaFree(g.tk_sp);
  g.tk_q = nullptr;
  g.tk_sp = nullptr;
  g.tk_K = 0;
  const size_t cnt = size_t(std::max(g.n, 1)) * 2 * K;
  cudaError_t e = cudaMalloc(&g.tk_q, cnt * sizeof(double2));
  if (e == cudaSuccess) e = cudaMalloc(&g.tk_sp, cnt * sizeof(int32_t));
  if (e == cudaSuccess && !g.tk_slack) e = cudaMalloc(&g.tk_slack, size_t(std::max(g.num_ep, 1)) * sizeof(double));
  if (e == cudaSuccess && !g.tk_star) e = cudaMalloc(&g.tk_star, size_t(std::max(g.num_ep, 1)) * 2 * sizeof(int32_t));
  if (e == cudaSuccess && !g.tk_summary) e = cudaMalloc(&g.tk_summary, 4 * sizeof(double));
  if (e != cudaSuccess) return int(e);
  g.tk_K = K;
  return 0;
}

template <int G>
static void launch_one(unsigned blocks, cudaStream_t st, const TkParams& P) {
  tk_one_kernel<G><<<blocks, 256, 0, st>>>(P);
}
template <int G>
static void launch_multi(unsigned blocks, cudaStream_t st, const TkParams& P) {
  tk_level_kernel<G><<<blocks, 256, 0, st>>>(P);
}

static void launch_g(bool one, int G, unsigned blocks, cudaStream_t st, const TkParams& P) {
  switch (G) {
    case 1: one ? launch_one<1>(blocks, st, P) : launch_multi<1>(blocks, st, P); break;
    case 2: one ? launch_one<2>(blocks, st, P) : launch_multi<2>(blocks, st, P); break;
    case 4: one ? launch_one<4>(blocks, st, P) : launch_multi<4>(blocks, st, P); break;
    case 8: one ? launch_one<8>(blocks, st, P) : launch_multi<8>(blocks, st, P); break;
    case 16: one ? launch_one<16>(blocks, st, P) : launch_multi<16>(blocks, st, P); break;
    default: one ? launch_one<32>(blocks, st, P) : launch_multi<32>(blocks, st, P); break;
  }
}

int launch_topk_forward(DevGraph& g, int K, float n_sigma, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  int err = ensure_topk(g, K);
  if (err) return err;
  if (g.n == 0) return 0;
  const long long ns = 2LL * g.num_src * K;
  if (ns > 0) tk_src_kernel<<<unsigned((ns + 255) / 256), 256, 0, st>>>(g.num_src, K, g.src_ms, g.tk_q, g.tk_sp);
  TkParams P;
  P.K = K;
  P.ns = double(n_sigma);
  P.list = g.tk_list;
  P.fanin_ptr = g.fanin_ptr;
  P.fin_src = g.fin_src;
  P.fin_ms = g.fin_ms;
  P.q = g.tk_q;
  P.qsp = g.tk_sp;
  if (K > 32) {   // wide queues: a warp per (pin, rf); single-arc pins, then the merging pins of a level
    for (int l = 1; l < g.num_levels; ++l) {
      P.lo = g.tk_one_ptr[l];
      P.hi = g.tk_multi_ptr[l];
      if (P.hi > P.lo)
        tk_one_wide_kernel<<<unsigned((2LL * (P.hi - P.lo) + kTkWideWarps - 1) / kTkWideWarps),
                             32 * kTkWideWarps, 0, st>>>(P);
      P.lo = g.tk_multi_ptr[l];
      P.hi = g.tk_one_ptr[l + 1];
      if (P.hi > P.lo)
        tk_wide_kernel<<<unsigned((2LL * (P.hi - P.lo) + kTkWideWarps - 1) / kTkWideWarps), 32 * kTkWideWarps, 0,
                         st>>>(P);
    }
    return int(cudaGetLastError());
  }
  const int G = pow2_group(K);
  // The two parts of a level are independent: the bandwidth-bound single-arc
  // kernel runs on a side stream next to the ALU-bound merging kernel on the
  // caller's stream; each waits for both parts of the previous level.
  cudaStream_t s2 = static_cast<cudaStream_t>(g.tk_side);
  cudaEvent_t* ev = reinterpret_cast<cudaEvent_t*>(g.tk_ev);
  cudaError_t e = cudaEventRecord(ev[0], st);   // sources written
  if (e == cudaSuccess) e = cudaStreamWaitEvent(s2, ev[0], 0);
  for (int l = 1; l < g.num_levels && e == cudaSuccess; ++l) {
    const bool has_one = g.tk_multi_ptr[l] > g.tk_one_ptr[l];
    const bool has_multi = g.tk_one_ptr[l + 1] > g.tk_multi_ptr[l];
    if (has_one) {
      P.lo = g.tk_one_ptr[l];
      P.hi = g.tk_multi_ptr[l];
      launch_g(true, G, unsigned((2LL * (P.hi - P.lo) * G + 255) / 256), s2, P);
      e = cudaEventRecord(ev[1], s2);
    }
    if (has_multi) {
      P.lo = g.tk_multi_ptr[l];
      P.hi = g.tk_one_ptr[l + 1];
      launch_g(false, G, unsigned((2LL * (P.hi - P.lo) * G + 255) / 256), st, P);
    }
    // join: the caller's stream waits for the side part; the side stream for the caller's
    if (e == cudaSuccess && has_one) e = cudaStreamWaitEvent(st, ev[1], 0);
    if (e == cudaSuccess && has_multi) e = cudaEventRecord(ev[0], st);
    if (e == cudaSuccess && has_multi) e = cudaStreamWaitEvent(s2, ev[0], 0);
  }
  if (e != cudaSuccess) return int(e);
  return int(cudaGetLastError());
}

int topk_stats(unsigned long long* out) {
#ifdef TK_STATS
  return int(cudaMemcpyFromSymbol(out, tk_stats, sizeof(unsigned long long) * 33));
#else
  (void)out;
  return -1;
#endif
}

int launch_topk_slack(DevGraph& g, float n_sigma, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (g.num_ep == 0) return int(cudaMemsetAsync(g.tk_summary, 0, 3 * sizeof(double), st));
  const long long threads = 32LL * g.num_ep;
  tk_slack_kernel<<<unsigned((threads + 255) / 256), 256, 0, st>>>(
      g.num_ep, g.tk_K, double(n_sigma), g.ep_pin, g.ep_rat, g.rat_ptr, g.rat_sp, g.rat_val, g.tk_q, g.tk_sp,
      g.tk_slack, g.tk_star);
  tk_reduce_kernel<<<1, 1024, 0, st>>>(g.num_ep, g.tk_slack, g.tk_summary);
  return int(cudaGetLastError());
}

int launch_topk_export(DevGraph& g, float* A, float* mean, float* sigma, int32_t* sp, void* stream) {
  const long long cnt = 2LL * g.n * g.tk_K;
  if (cnt == 0) return 0;
  tk_export_kernel<<<unsigned((cnt + 255) / 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(
      g.n, g.tk_K, double(g.tk_ns), g.order, g.tk_q, g.tk_sp, A, mean, sigma, sp);
  return int(cudaGetLastError());
}

int launch_topk_export_slack(DevGraph& g, float* slack, int32_t* sp_star, uint8_t* rf_star, int32_t* k_star,
                             void* stream) {
  if (g.num_ep == 0) return 0;
  tk_export_slack_kernel<<<(g.num_ep + 255) / 256, 256, 0, static_cast<cudaStream_t>(stream)>>>(
      g.num_ep, g.order, g.tk_slack, g.tk_star, slack, sp_star, rf_star, k_star);
  return int(cudaGetLastError());
}

}  // namespace insta
