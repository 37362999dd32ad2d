// slack_common.cuh -- endpoint slack + WNS/TNS (Eq 3
// corner arrival): slack = RAT - A, min over rf (tie -> R); TNS / WNS /
// violation count in fp64 with a fixed reduction order.  Shared by
// slack_kernel (kernels.cu) and the candidate-evaluation kernel (sweep.cu), so
// that a block's partial recomputed there is bit-identical to slack_kernel's.
//
// Layout: nb blocks of kRedThreads logical threads; logical thread t of block
// b sums endpoints k = b * kRedThreads + t + j * nb * kRedThreads in index
// order; warp and block trees in a fixed order -> partials[3 b .. 3 b + 2]
// {tns, wns, nv}; the final reduction walks the partials with the same fixed
// strides.  The physical CTA may be wider than kRedThreads (extra threads idle).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "device_common.cuh"
#include "internal.h"

namespace insta {

constexpr int kRedThreads = 256;
constexpr int kRedBlocksPerSM = 4;   // slack grid: a fixed multiple of the SM count (fixed summation order)

__device__ __forceinline__ Gath load_state_plain(const PinState* p) {
  const double2 m = __ldcg(reinterpret_cast<const double2*>(p));
  const double2 v = __ldcg(reinterpret_cast<const double2*>(p) + 1);
  Gath g;
  g.mu0 = strip((unsigned long long)__double_as_longlong(m.x));
  g.mu1 = strip((unsigned long long)__double_as_longlong(m.y));
  g.v0 = strip((unsigned long long)__double_as_longlong(v.x));
  g.v1 = strip2((unsigned long long)__double_as_longlong(v.y));
  return g;
}

// warp reduction in a fixed order (deterministic): sum / min of fp64
__device__ __forceinline__ double warp_sum(double v) {
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ double warp_min(double v) {
  for (int o = 16; o > 0; o >>= 1) v = fmin(v, __shfl_down_sync(0xffffffffu, v, o));
  return v;
}

struct SlackRed {
  double r[3][kRedThreads / 32];
};

// Block b's partial (every thread of the CTA calls it; it holds __syncthreads).
__device__ __forceinline__ void slack_block(int b, int nb, int num_ep, const int32_t* __restrict__ ep_pin,
                                            const float2* __restrict__ ep_rat, const PinState* state, double ns,
                                            float* slack, uint8_t* rf_star, double* partials, SlackRed& sr) {
  double tns = 0.0, wns = 0.0, nv = 0.0;
  const int t = threadIdx.x;
  if (t < kRedThreads) {
    for (int k = b * kRedThreads + t; k < num_ep; k += nb * kRedThreads) {
      const Gath st = load_state_plain(state + ep_pin[k]);
      const float2 rat = ep_rat[k];
      const double sR = double(rat.x) - (st.mu0 + ns * double(sigma_of(st.v0)));   // Eq 3 corner
      const double sF = double(rat.y) - (st.mu1 + ns * double(sigma_of(st.v1)));
      const bool fall = sF < sR;
      const double sv = fall ? sF : sR;
      slack[k] = float(sv);
      rf_star[k] = fall ? 1 : 0;
      if (sv < 0.0) {
        tns += sv;
        nv += 1.0;
        wns = fmin(wns, sv);
      }
    }
  }
  const int w = t >> 5, lane = t & 31;
  if (t < kRedThreads) {
    tns = warp_sum(tns);
    wns = warp_min(wns);
    nv = warp_sum(nv);
    if (lane == 0) {
      sr.r[0][w] = tns;
      sr.r[1][w] = wns;
      sr.r[2][w] = nv;
    }
  }
  __syncthreads();
  if (w == 0) {
    tns = lane < kRedThreads / 32 ? sr.r[0][lane] : 0.0;
    wns = lane < kRedThreads / 32 ? sr.r[1][lane] : 0.0;
    nv = lane < kRedThreads / 32 ? sr.r[2][lane] : 0.0;
    tns = warp_sum(tns);
    wns = warp_min(wns);
    nv = warp_sum(nv);
    if (lane == 0) {
      partials[3 * b + 0] = tns;
      partials[3 * b + 1] = wns;
      partials[3 * b + 2] = nv;
    }
  }
  __syncthreads();
}

// {wns, tns, nv} over the nb partials (every thread of the CTA calls it; written by thread 0)
__device__ __forceinline__ void slack_final(int nb, const double* partials, double* out, SlackRed& sr) {
  const int t = threadIdx.x, w = t >> 5, lane = t & 31;
  double tns = 0.0, wns = 0.0, nv = 0.0;
  if (t < kRedThreads) {
    for (int b = t; b < nb; b += kRedThreads) {
      tns += __ldcg(partials + 3 * b + 0);
      wns = fmin(wns, __ldcg(partials + 3 * b + 1));
      nv += __ldcg(partials + 3 * b + 2);
    }
    tns = warp_sum(tns);
    wns = warp_min(wns);
    nv = warp_sum(nv);
    if (lane == 0) {
      sr.r[0][w] = tns;
      sr.r[1][w] = wns;
      sr.r[2][w] = nv;
    }
  }
  __syncthreads();
  if (t == 0) {
    tns = 0.0;
    wns = 0.0;
    nv = 0.0;
    for (int k = 0; k < kRedThreads / 32; ++k) {
      tns += sr.r[0][k];
      wns = fmin(wns, sr.r[1][k]);
      nv += sr.r[2][k];
    }
    out[0] = wns;
    out[1] = tns;
    out[2] = nv;
  }
  __syncthreads();
}

// the slack grid's block count for num_ep endpoints on a device with sms SMs
inline int slack_blocks(int num_ep, int sms) {
  const int b = (num_ep + kRedThreads - 1) / kRedThreads;
  const int cap = kRedBlocksPerSM * sms;
  return b < 1 ? 1 : (b < cap ? b : cap);
}

}  // namespace insta
