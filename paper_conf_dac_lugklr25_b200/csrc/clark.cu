// clark.cu -- Clark moment-matching statistical max: the
// merge the north star names beside the paper's smooth max (Eq 4).
//
// A pin's arrival per transition rf is the Gaussian (mu, V = sigma^2).  A
// candidate through fanin arc e = (j -> i) and source transition s is
// (mu_j[s] + mean_e[rf], V_j[s] + std_e[rf]^2) (Eq 1-2); the merge folds the
// candidates in canonical order (fanin row = caller arc id order, then s = rf
// before ~rf) with Clark's max of two independent Gaussians (R20):
//   a = sqrt(V1 + V2), alpha = (mu1 - mu2) / a
//   mu = mu1 Phi(alpha) + mu2 Phi(-alpha) + a phi(alpha)
//   V  = (mu1^2 + V1) Phi(alpha) + (mu2^2 + V2) Phi(-alpha) + (mu1 + mu2) a phi(alpha) - mu^2
// (a = 0: the hard max, first input wins ties).  Endpoints: A = mu + N_sigma
// sqrt(V) (Eq 3), slack as in insta_slack.
//
// Execution: per-level launches, a thread per (pin, rf), fp64 throughout.
// The forward stores the prefix of the fold after every candidate, so the
// backward (reverse levels) only evaluates Clark's Jacobian at (prefix,
// candidate).  Adjoints flow pull-style without atomics: a sink writes one
// adjoint slot per (fanin position, sink rf, source-transition index); a
// source sums its fanout slots in fanout order -- deterministic.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <vector>

#include "device_common.cuh"
#include "internal.h"

namespace insta {

struct ClParams {
  int32_t lo, hi;
  double ns;
  const int32_t* __restrict__ fanin_ptr;
  const int32_t* __restrict__ fin_src;
  const float4* __restrict__ fin_ms;
  const int32_t* __restrict__ fin_arc;   // caller arc id per fanin position
  const int32_t* __restrict__ fo_ptr;    // [n+1] full fanout rows (canonical)
  const int32_t* __restrict__ fo_q;      // fanout word: fanin position << 2 | unateness
  const float4* __restrict__ src_ms;
  const int32_t* __restrict__ ep_of_pin;
  double2* mv;        // [n][2] {mu, V}
  double2* pre;       // [e][2 sink rf][2 s index] prefix of the fold after the candidate
  double2* g;         // [e][2 sink rf][2 s index] adjoint {mubar, Vbar} of the candidate
  const double* slack;
  const uint8_t* rf_star;
  const float* ep_seed;   // NULL = TNS
  float* d_mean;
  float* d_sigma;
  float* d_src;           // [n][2] caller order or NULL
  const int32_t* __restrict__ order;
  // wide-fanout pins of the level (cl_pull_wide_kernel)
  int32_t hv_lo, hv_hi;
  const int32_t* __restrict__ hv_list;   // canonical pins, grouped by level
  const int32_t* __restrict__ hv_of;     // [n] index into hv_list / hv_sum, -1 = narrow
  double2* hv_sum;                       // [num wide][2] pulled adjoints
};

__device__ __forceinline__ double cl_pdf(double x) { return exp(-0.5 * x * x) * 0.39894228040143267794; }

__device__ __forceinline__ void clark2(double m1, double v1, double m2, double v2, double& m, double& v) {
  const double a2 = v1 + v2;
  if (!(a2 > 0.0)) {
    if (m2 > m1) {
      m = m2;
      v = v2;
    } else {
      m = m1;
      v = v1;
    }
    return;
  }
  const double a = sqrt(a2), al = (m1 - m2) / a;
  const double P = normcdf(al), Q = normcdf(-al), p = cl_pdf(al);
  m = m1 * P + m2 * Q + a * p;
  const double e2 = (m1 * m1 + v1) * P + (m2 * m2 + v2) * Q + (m1 + m2) * a * p;
  v = fmax(e2 - m * m, 0.0);
}

// Jacobian rows d(mu)/d(m1, v1, m2, v2) and d(V)/d(...)
__device__ __forceinline__ void clark2_jac(double m1, double v1, double m2, double v2, double Jm[4], double Jv[4]) {
  const double a2 = v1 + v2;
  if (!(a2 > 0.0)) {
    const bool second = m2 > m1;
    for (int c = 0; c < 4; ++c) Jm[c] = Jv[c] = 0.0;
    Jm[second ? 2 : 0] = 1.0;
    Jv[second ? 3 : 1] = 1.0;
    return;
  }
  const double a = sqrt(a2), al = (m1 - m2) / a;
  const double P = normcdf(al), Q = normcdf(-al), p = cl_pdf(al);
  const double mu = m1 * P + m2 * Q + a * p;
  const double dv = p / (2.0 * a);
  const double e_m1 = 2.0 * m1 * P + a * p + (p / a) * (v1 - v2);
  const double e_m2 = 2.0 * m2 * Q + a * p - (p / a) * (v1 - v2);
  const double e_a = (m1 + m2) * p - al * p * (v1 - v2) / a;
  Jm[0] = P;
  Jm[1] = dv;
  Jm[2] = Q;
  Jm[3] = dv;
  Jv[0] = e_m1 - 2.0 * mu * P;
  Jv[1] = P + e_a / (2.0 * a) - 2.0 * mu * dv;
  Jv[2] = e_m2 - 2.0 * mu * Q;
  Jv[3] = Q + e_a / (2.0 * a) - 2.0 * mu * dv;
}

// candidate (q, si) of sink transition rf
__device__ __forceinline__ double2 cl_cand(const ClParams& P, int q, int rf, int si) {
  const int32_t w = __ldg(P.fin_src + q);
  const float4 ms = __ldg(P.fin_ms + q);
  const int s = src_tr(rf, int(uint32_t(w) >> kUnateShift), si);
  const double2 st = P.mv[size_t(w & kSrcMask) * 2 + s];
  const double sd = double(rf ? ms.w : ms.z);
  return make_double2(st.x + double(rf ? ms.y : ms.x), st.y + sd * sd);   // Eq 1-2
}

__global__ void cl_fwd_kernel(ClParams P) {
  const long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (x >= 2LL * (P.hi - P.lo)) return;
  const int i = P.lo + int(x >> 1), rf = int(x & 1);
  const int b0 = __ldg(P.fanin_ptr + i), b1 = __ldg(P.fanin_ptr + i + 1);
  double m = 0.0, v = 0.0;
  if (b0 == b1) {   // startpoint
    const float4 s = __ldg(P.src_ms + i);
    const double sd = double(rf ? s.w : s.z);
    m = double(rf ? s.y : s.x);
    v = sd * sd;
  } else {
    bool first = true;
    for (int q = b0; q < b1; ++q) {
      const int u = int(uint32_t(__ldg(P.fin_src + q)) >> kUnateShift);
      for (int si = 0; si < n_src_tr(u); ++si) {
        const double2 c = cl_cand(P, q, rf, si);
        if (first) {
          m = c.x;
          v = c.y;
          first = false;
        } else {
          clark2(m, v, c.x, c.y, m, v);
        }
        P.pre[(size_t(q) * 2 + rf) * 2 + si] = make_double2(m, v);
      }
    }
  }
  P.mv[size_t(i) * 2 + rf] = make_double2(m, v);
}

// endpoint slack (rf tie -> R) in fp64
__global__ void cl_slack_kernel(int num_ep, double ns, const int32_t* __restrict__ ep_pin, const float2* __restrict__ ep_rat,
                                const double2* __restrict__ mv, double* slack, uint8_t* rf_star) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= num_ep) return;
  const int p = __ldg(ep_pin + e);
  const float2 r = __ldg(ep_rat + e);
  const double2 a = mv[size_t(p) * 2], b = mv[size_t(p) * 2 + 1];
  const double sr = double(r.x) - (a.x + ns * sqrt(a.y));
  const double sf = double(r.y) - (b.x + ns * sqrt(b.y));
  const bool f = sf < sr;
  slack[e] = f ? sf : sr;
  rf_star[e] = f ? 1 : 0;
}

__global__ void __launch_bounds__(1024) cl_reduce_kernel(int num_ep, const double* __restrict__ slack, double* out) {
  __shared__ double s_t[1024], s_w[1024], s_n[1024];
  const int t = threadIdx.x;
  double tns = 0.0, wns = 0.0, nv = 0.0;
  // thread t sums endpoints t, t + 1024, ... (coalesced; four loads in flight), fixed order
  for (int e0 = t; e0 < num_ep; e0 += 4 * 1024) {
    double v[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) v[j] = e0 + j * 1024 < num_ep ? slack[e0 + j * 1024] : 0.0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (v[j] < 0.0) {
        tns += v[j];
        nv += 1.0;
      }
      wns = fmin(wns, v[j]);
    }
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

// Backward of one level: (1) pull the adjoint of (pin, rf) from the slots its
// fanout sinks wrote (+ the endpoint seed); (2) reverse the fold with Clark's
// Jacobian at (prefix, candidate) and write each candidate's adjoint slot and
// the arc gradients.
// Sum of the candidate adjoints a pin's fanout sinks wrote for its transition
// rf over fanout entries k0, k0 + step, ...  Fanout word = fanin position << 2 |
// unateness; the slots feeding source transition rf: POS (rf, 0); NEG (~rf,
// 0); NON (rf, 0) and (~rf, 1).  Four entries per round keep loads in flight.
__device__ __forceinline__ double2 cl_pull(const ClParams& P, int rf, int k0, int k1, int step) {
  double um = 0.0, uv = 0.0;
  for (int kb = k0; kb < k1; kb += 4 * step) {
    uint32_t w[4];
#pragma unroll
    for (int t = 0; t < 4; ++t) w[t] = kb + t * step < k1 ? uint32_t(__ldg(P.fo_q + kb + t * step)) : 0xffffffffu;
    double2 g0[4], g1[4];
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      g0[t] = make_double2(0.0, 0.0);
      g1[t] = make_double2(0.0, 0.0);
      if (w[t] != 0xffffffffu) {
        const size_t q = w[t] >> 2;
        const int u = int(w[t] & 3u);
        g0[t] = P.g[(q * 2 + (u == 1 ? rf ^ 1 : rf)) * 2];
        if (u == 2) g1[t] = P.g[(q * 2 + (rf ^ 1)) * 2 + 1];
      }
    }
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      um += g0[t].x;
      uv += g0[t].y;
      um += g1[t].x;
      uv += g1[t].y;
    }
  }
  return make_double2(um, uv);
}

// Pins with a wide fanout row (> kClWide): a warp per (pin, rf) pulls the row
// (lanes strided, fixed shuffle tree) into hv_sum before the level's fold kernel.
// A CTA of kClPullThreads per (pin, rf): thread t sums entries t, t + 128, ... in row order, then a
// fixed shuffle tree per warp and the warps in order -- deterministic; a 20k-sink net takes ~160
// rounds of one thread instead of ~625 of one warp lane (the warp-per-pin pull was 1.8 of the 6.1 ms
// backward at C4).
constexpr int kClWide = 32;
constexpr int kClPullThreads = 128;
__global__ void __launch_bounds__(kClPullThreads) cl_pull_wide_kernel(ClParams P) {
  __shared__ double2 s_w[kClPullThreads / 32];
  const long long x = blockIdx.x;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (x >= 2LL * (P.hv_hi - P.hv_lo)) return;
  const int h = P.hv_lo + int(x >> 1), rf = int(x & 1);
  const int i = __ldg(P.hv_list + h);
  double2 s = cl_pull(P, rf, __ldg(P.fo_ptr + i) + int(threadIdx.x), __ldg(P.fo_ptr + i + 1), kClPullThreads);
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) {
    s.x += __shfl_down_sync(0xffffffffu, s.x, d);
    s.y += __shfl_down_sync(0xffffffffu, s.y, d);
  }
  if (lane == 0) s_w[warp] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double2 t = s_w[0];
    for (int w = 1; w < kClPullThreads / 32; ++w) {
      t.x += s_w[w].x;
      t.y += s_w[w].y;
    }
    P.hv_sum[size_t(h) * 2 + rf] = t;
  }
}

// Backward of one level, a thread per (pin, rf): (1) the adjoint of (pin, rf)
// = the pulled fanout slots (+ the endpoint seed); (2) reverse the fold with
// Clark's Jacobian at (prefix, candidate), write each candidate's adjoint slot
// and the arc gradients.
#ifndef CL_BWD_MINB
#define CL_BWD_MINB 4   // resident 256-thread blocks per SM (<= 64 registers): latency-bound gathers want warps
#endif
__global__ void __launch_bounds__(256, CL_BWD_MINB) cl_bwd_kernel(ClParams P) {
  const long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (x >= 2LL * (P.hi - P.lo)) return;
  const int i = P.lo + int(x >> 1), rf = int(x & 1);
  const int hv = __ldg(P.hv_of + i);
  const double2 pulled = hv >= 0 ? P.hv_sum[size_t(hv) * 2 + rf]
                                 : cl_pull(P, rf, __ldg(P.fo_ptr + i), __ldg(P.fo_ptr + i + 1), 1);
  double um = pulled.x, uv = pulled.y;
  const int ep = __ldg(P.ep_of_pin + i);
  if (ep >= 0 && P.rf_star[ep] == rf) {
    const double s = P.slack[ep];
    const double seed = P.ep_seed ? double(P.ep_seed[ep]) : (s < 0.0 ? 1.0 : 0.0);
    const double V = P.mv[size_t(i) * 2 + rf].y;
    um += -seed;
    uv += V > 0.0 ? -seed * P.ns / (2.0 * sqrt(V)) : 0.0;
  }
  const int b0 = __ldg(P.fanin_ptr + i), b1 = __ldg(P.fanin_ptr + i + 1);
  if (b0 == b1) {
    if (P.d_src) P.d_src[size_t(__ldg(P.order + i)) * 2 + rf] = float(um);
    return;
  }
  // reverse over the candidates: (q, si) from the last to the first
  int q = b1 - 1;
  int si = n_src_tr(int(uint32_t(__ldg(P.fin_src + q)) >> kUnateShift)) - 1;
  double am = 0.0, asg = 0.0;   // per-arc sums over si for the current q
  while (true) {
    int pq = q, psi = si - 1;   // previous candidate in the fold order
    if (psi < 0) {
      pq = q - 1;
      psi = pq >= b0 ? n_src_tr(int(uint32_t(__ldg(P.fin_src + pq)) >> kUnateShift)) - 1 : -1;
    }
    double cm, cv;
    if (pq >= b0) {
      const double2 pr = P.pre[(size_t(pq) * 2 + rf) * 2 + psi];
      const double2 c = cl_cand(P, q, rf, si);
      double Jm[4], Jv[4];
      clark2_jac(pr.x, pr.y, c.x, c.y, Jm, Jv);
      cm = um * Jm[2] + uv * Jv[2];
      cv = um * Jm[3] + uv * Jv[3];
      const double nm = um * Jm[0] + uv * Jv[0];
      const double nv = um * Jm[1] + uv * Jv[1];
      um = nm;
      uv = nv;
    } else {   // the first candidate takes what is left
      cm = um;
      cv = uv;
    }
    P.g[(size_t(q) * 2 + rf) * 2 + si] = make_double2(cm, cv);
    am += cm;
    asg += cv;
    if (si == 0) {   // all candidates of arc q done: its gradients (inputs of Eq 1-2)
      const float4 ms = __ldg(P.fin_ms + q);
      const size_t arc = size_t(__ldg(P.fin_arc + q));
      P.d_mean[arc * 2 + rf] = float(am);
      if (P.d_sigma) P.d_sigma[arc * 2 + rf] = float(2.0 * double(rf ? ms.w : ms.z) * asg);
      am = 0.0;
      asg = 0.0;
    }
    if (pq < b0) break;
    q = pq;
    si = psi;
  }
}

// --------------------------------------------------------------------------
// host launchers
// --------------------------------------------------------------------------
// Full fanout rows (heavy drivers included) as words fanin position << 2 |
// unateness, and the wide-fanout pins per level; shared by the Clark backward
// and the Eq 7 gradient (place.cu).
int ensure_fanout_words(DevGraph& g) {
  if (g.cl_fo_q) return 0;
  const HostLevels& h = g.host;
  std::vector<int32_t> fo_q(size_t(std::max<int64_t>(g.e, 1)));
  std::vector<int32_t> fsrc(size_t(std::max<int64_t>(g.e, 1)));
  if (g.e > 0) {
    cudaError_t e0 = cudaMemcpy(fsrc.data(), g.fin_src, sizeof(int32_t) * size_t(g.e), cudaMemcpyDeviceToHost);
    if (e0 != cudaSuccess) return int(e0);
  }
  if (g.e >= (int64_t(1) << 30)) return int(cudaErrorInvalidValue);
  for (int64_t k = 0; k < g.e; ++k) {
    const int32_t q = g.h_arc_pos[size_t(h.fanout_arc[size_t(k)])];
    fo_q[size_t(k)] = int32_t((uint32_t(q) << 2) | (uint32_t(fsrc[size_t(q)]) >> kUnateShift));
  }
  // wide-fanout pins per level
  std::vector<int32_t> hv_list, hv_of(size_t(std::max(g.n, 1)), -1);
  g.cl_hv_ptr.assign(size_t(g.num_levels) + 1, 0);
  for (int l = 0; l < g.num_levels; ++l) {
    g.cl_hv_ptr[l] = int32_t(hv_list.size());
    for (int p = h.level_ptr[l]; p < h.level_ptr[l + 1]; ++p)
      if (h.fanout_ptr[p + 1] - h.fanout_ptr[p] > kClWide) {
        hv_of[size_t(p)] = int32_t(hv_list.size());
        hv_list.push_back(p);
      }
  }
  g.cl_hv_ptr[g.num_levels] = int32_t(hv_list.size());
  cudaError_t e = cudaMalloc(&g.cl_hv_list, sizeof(int32_t) * std::max<size_t>(hv_list.size(), 1));
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_hv_of, sizeof(int32_t) * hv_of.size());
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_hv_sum, sizeof(double2) * 2 * std::max<size_t>(hv_list.size(), 1));
  if (e == cudaSuccess && !hv_list.empty())
    e = cudaMemcpy(g.cl_hv_list, hv_list.data(), sizeof(int32_t) * hv_list.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(g.cl_hv_of, hv_of.data(), sizeof(int32_t) * hv_of.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_fo_ptr, sizeof(int32_t) * (size_t(g.n) + 1));
  if (e == cudaSuccess)
    e = cudaMemcpy(g.cl_fo_ptr, h.fanout_ptr.data(), sizeof(int32_t) * (size_t(g.n) + 1), cudaMemcpyHostToDevice);
  int32_t* fq = nullptr;
  if (e == cudaSuccess) e = cudaMalloc(&fq, sizeof(int32_t) * fo_q.size());
  if (e == cudaSuccess) e = cudaMemcpy(fq, fo_q.data(), sizeof(int32_t) * fo_q.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) g.cl_fo_q = fq;
  return int(e);
}

static int ensure_clark(DevGraph& g) {
  if (g.cl_mv) return 0;
  int err = ensure_fanout_words(g);
  if (err) return err;
  cudaError_t e = cudaMalloc(&g.cl_mv, sizeof(double2) * 2 * size_t(std::max(g.n, 1)));
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_pre, sizeof(double2) * 4 * size_t(std::max<int64_t>(g.e, 1)));
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_g, sizeof(double2) * 4 * size_t(std::max<int64_t>(g.e, 1)));
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_slack, sizeof(double) * size_t(std::max(g.num_ep, 1)));
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_rf, size_t(std::max(g.num_ep, 1)));
  if (e == cudaSuccess) e = cudaMalloc(&g.cl_summary, 4 * sizeof(double));
  return int(e);
}

static ClParams cl_params(DevGraph& g, float n_sigma) {
  ClParams P{};
  P.ns = double(n_sigma);
  P.fanin_ptr = g.fanin_ptr;
  P.fin_src = g.fin_src;
  P.fin_ms = g.fin_ms;
  P.fin_arc = g.fin_arc;
  P.fo_ptr = g.cl_fo_ptr;
  P.fo_q = g.cl_fo_q;
  P.src_ms = g.src_ms;
  P.ep_of_pin = g.ep_of_pin;
  P.mv = reinterpret_cast<double2*>(g.cl_mv);
  P.pre = reinterpret_cast<double2*>(g.cl_pre);
  P.g = reinterpret_cast<double2*>(g.cl_g);
  P.slack = g.cl_slack;
  P.rf_star = g.cl_rf;
  P.order = g.order;
  P.hv_list = g.cl_hv_list;
  P.hv_of = g.cl_hv_of;
  P.hv_sum = reinterpret_cast<double2*>(g.cl_hv_sum);
  return P;
}

int launch_clark_forward(DevGraph& g, float n_sigma, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  int err = ensure_clark(g);
  if (err) return err;
  ClParams P = cl_params(g, n_sigma);
  const std::vector<int32_t>& lp = g.host.level_ptr;
  for (int l = 0; l < g.num_levels; ++l) {
    P.lo = lp[l];
    P.hi = lp[l + 1];
    const long long threads = 2LL * (P.hi - P.lo);
    if (threads > 0) cl_fwd_kernel<<<unsigned((threads + 255) / 256), 256, 0, st>>>(P);
  }
  if (g.num_ep > 0) {
    cl_slack_kernel<<<(g.num_ep + 255) / 256, 256, 0, st>>>(g.num_ep, double(n_sigma), g.ep_pin, g.ep_rat,
                                                            reinterpret_cast<const double2*>(g.cl_mv), g.cl_slack,
                                                            g.cl_rf);
    cl_reduce_kernel<<<1, 1024, 0, st>>>(g.num_ep, g.cl_slack, g.cl_summary);
  } else {
    cudaMemsetAsync(g.cl_summary, 0, 3 * sizeof(double), st);
  }
  return int(cudaGetLastError());
}

int launch_clark_backward(DevGraph& g, const float* ep_seed, float* d_mean, float* d_sigma, float* d_src,
                          void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  ClParams P = cl_params(g, g.cl_ns);
  P.ep_seed = ep_seed;
  P.d_mean = d_mean;
  P.d_sigma = d_sigma;
  P.d_src = d_src;
  if (d_src) {
    cudaError_t e = cudaMemsetAsync(d_src, 0, sizeof(float) * 2 * size_t(g.n), st);
    if (e != cudaSuccess) return int(e);
  }
  const std::vector<int32_t>& lp = g.host.level_ptr;
  for (int l = g.num_levels - 1; l >= 0; --l) {
    P.lo = lp[l];
    P.hi = lp[l + 1];
    P.hv_lo = g.cl_hv_ptr[l];
    P.hv_hi = g.cl_hv_ptr[l + 1];
    if (P.hv_hi > P.hv_lo)   // a CTA per (wide pin, rf)
      cl_pull_wide_kernel<<<unsigned(2LL * (P.hv_hi - P.hv_lo)), kClPullThreads, 0, st>>>(P);
    const long long threads = 2LL * (P.hi - P.lo);
    if (threads > 0) cl_bwd_kernel<<<unsigned((threads + 255) / 256), 256, 0, st>>>(P);
  }
  return int(cudaGetLastError());
}

__global__ void cl_export_kernel(int n, double ns, const int32_t* __restrict__ order, const double2* __restrict__ mv,
                                 float* A, float* mean, float* sigma) {
  const long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (x >= 2LL * n) return;
  const size_t o = size_t(__ldg(order + int(x >> 1))) * 2 + size_t(x & 1);
  const double2 v = mv[x];
  const double sg = sqrt(v.y);
  if (A) A[o] = float(v.x + ns * sg);
  if (mean) mean[o] = float(v.x);
  if (sigma) sigma[o] = float(sg);
}

__global__ void cl_export_slack_kernel(int num_ep, const double* __restrict__ slack, const uint8_t* __restrict__ rf,
                                       float* out, uint8_t* rf_out) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= num_ep) return;
  if (out) out[e] = float(slack[e]);
  if (rf_out) rf_out[e] = rf[e];
}

int launch_clark_export(DevGraph& g, float* A, float* mean, float* sigma, float* slack, uint8_t* rf, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if ((A || mean || sigma) && g.n > 0)
    cl_export_kernel<<<unsigned((2LL * g.n + 255) / 256), 256, 0, st>>>(
        g.n, double(g.cl_ns), g.order, reinterpret_cast<const double2*>(g.cl_mv), A, mean, sigma);
  if ((slack || rf) && g.num_ep > 0)
    cl_export_slack_kernel<<<(g.num_ep + 255) / 256, 256, 0, st>>>(g.num_ep, g.cl_slack, g.cl_rf, slack, rf);
  return int(cudaGetLastError());
}

}  // namespace insta
