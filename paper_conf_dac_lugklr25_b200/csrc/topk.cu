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

namespace insta {

struct TkParams {
  int32_t lo, hi, K;
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

template <int G>
__global__ void __launch_bounds__(256) tk_level_kernel(TkParams P) {
  const int lane = threadIdx.x & 31;
  const int gl = lane & (G - 1), gbase = lane & ~(G - 1);
  const unsigned gm = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << gbase);
  const long long grp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) / G;
  if (grp >= 2LL * (P.hi - P.lo)) return;   // uniform within a group
  const int i = P.lo + int(grp >> 1), rf = int(grp & 1), K = P.K;
  const bool slot = gl < K;
  const int last = gbase + K - 1;
  double qA = -INFINITY, qmu = 0.0, qvar = 0.0;
  int qsp = -1, qt = INT_MAX;
  const int b0 = __ldg(P.fanin_ptr + i), b1 = __ldg(P.fanin_ptr + i + 1), nf = b1 - b0;
  for (int a = b0; a < b1; ++a) {
    const int32_t w = __ldg(P.fin_src + a);
    const int j = w & kSrcMask, u = int(uint32_t(w) >> kUnateShift);
    const float4 ms = __ldg(P.fin_ms + a);
    const double am = double(rf ? ms.y : ms.x), se = double(rf ? ms.w : ms.z);
    for (int si = 0; si < n_src_tr(u); ++si) {
      const size_t ps = (size_t(j) * 2 + src_tr(rf, u, si)) * K + gl;
      const int csp = slot ? __ldg(P.qsp + ps) : -1;
      double cA = -INFINITY, cmu = 0.0, cvar = 0.0;
      const int ct = (gl * nf + (a - b0)) * 2 + si;   // Alg 1 order: k outer, arcs, s
      if (csp >= 0) {
        const double2 pv = __ldg(P.q + ps);
        cmu = pv.x + am;                               // Eq 1 (l.12)
        cvar = pv.y + se * se;                         // Eq 2 (l.13)
        cA = cmu + P.ns * double(sigma_of(cvar));      // Eq 3 (l.14)
      }
      if (a == b0 && si == 0) {
        // first batch into an empty queue: one parent's queue has unique
        // startpoints, so Alg 2 reduces to ordering the candidates by key --
        // a bitonic sort over the group (skipped when already in order)
        const double nA = __shfl_down_sync(gm, cA, 1, G);
        const int nt = __shfl_down_sync(gm, ct, 1, G);
        const bool bad = gl + 1 < G && key_gt(nA, nt, cA, ct);
        int idx = gl;
        if (__ballot_sync(gm, bad) & gm) {
          double sA = cA;
          int st = csp >= 0 ? ct : INT_MAX;
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
        qA = __shfl_sync(gm, cA, gbase + idx);
        qmu = __shfl_sync(gm, cmu, gbase + idx);
        qvar = __shfl_sync(gm, cvar, gbase + idx);
        qsp = __shfl_sync(gm, csp, gbase + idx);
        qt = __shfl_sync(gm, ct, gbase + idx);
        if (qsp < 0) {
          qA = -INFINITY;
          qt = INT_MAX;
        }
        continue;
      }
      // one ballot prunes everything below the queue's last slot
      const double mA = __shfl_sync(gm, qA, last);
      const int mt = __shfl_sync(gm, qt, last);
      unsigned m = __ballot_sync(gm, csp >= 0 && key_gt(cA, ct, mA, mt)) & gm;
      while (m) {                                      // Alg 2 for each survivor
        const int src = __ffs(m) - 1;
        m &= m - 1;
        const double nA = __shfl_sync(gm, cA, src), nmu = __shfl_sync(gm, cmu, src),
                     nvar = __shfl_sync(gm, cvar, src);
        const int nt = __shfl_sync(gm, ct, src), nsp = __shfl_sync(gm, csp, src);
        const unsigned fm = __ballot_sync(gm, slot && qsp == nsp) & gm;
        int f;
        if (fm) {                                      // Step 1: the startpoint is queued
          f = __ffs(fm) - 1;
          if (!key_gt(nA, nt, __shfl_sync(gm, qA, f), __shfl_sync(gm, qt, f))) continue;
          f -= gbase;
        } else {                                       // Step 2: new startpoint
          if (!key_gt(nA, nt, __shfl_sync(gm, qA, last), __shfl_sync(gm, qt, last))) continue;
          f = K - 1;                                   // the last entry falls off
        }
        const int p = __popc(__ballot_sync(gm, slot && key_gt(qA, qt, nA, nt)) & gm);
        const double uA = __shfl_up_sync(gm, qA, 1, G), umu = __shfl_up_sync(gm, qmu, 1, G),
                     uvar = __shfl_up_sync(gm, qvar, 1, G);
        const int usp = __shfl_up_sync(gm, qsp, 1, G), ut = __shfl_up_sync(gm, qt, 1, G);
        if (gl > p && gl <= f) {
          qA = uA; qmu = umu; qvar = uvar; qsp = usp; qt = ut;
        } else if (gl == p) {
          qA = nA; qmu = nmu; qvar = nvar; qsp = nsp; qt = nt;
        }
      }
    }
  }
  if (slot) {
    const size_t o = (size_t(i) * 2 + rf) * K + gl;
    P.q[o] = make_double2(qmu, qvar);
    P.qsp[o] = qsp;
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
  P.fanin_ptr = g.fanin_ptr;
  P.fin_src = g.fin_src;
  P.fin_ms = g.fin_ms;
  P.q = g.tk_q;
  P.qsp = g.tk_sp;
  const int G = pow2_group(K);
  const std::vector<int32_t>& lp = g.host.level_ptr;
  for (int l = 1; l < g.num_levels; ++l) {
    P.lo = lp[l];
    P.hi = lp[l + 1];
    const long long threads = 2LL * (P.hi - P.lo) * G;
    const unsigned blocks = unsigned((threads + 255) / 256);
    switch (G) {
      case 1: tk_level_kernel<1><<<blocks, 256, 0, st>>>(P); break;
      case 2: tk_level_kernel<2><<<blocks, 256, 0, st>>>(P); break;
      case 4: tk_level_kernel<4><<<blocks, 256, 0, st>>>(P); break;
      case 8: tk_level_kernel<8><<<blocks, 256, 0, st>>>(P); break;
      case 16: tk_level_kernel<16><<<blocks, 256, 0, st>>>(P); break;
      default: tk_level_kernel<32><<<blocks, 256, 0, st>>>(P); break;
    }
  }
  return int(cudaGetLastError());
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
