// place.cu -- the device-side part of INSTA-Place:
// the timing objective of Eq 7,
//   L = lambda_RC * sum_k (|x_f - x_t| + |y_f - y_t|) * w_k,
// over every timing arc k = (f -> t) with a per-arc weight w_k (DESIGN.md
// R21: the arc's timing sensitivity, e.g. -(dTNS/dmean_R + dTNS/dmean_F) from
// insta_backward; 0 = not critical), its gradient w.r.t. the pin positions
// (subgradient sign(0) = 0), and the gradient-norm ratio of Eq 8.
//
// Loss: a thread per fanin position, fixed-order block tree + one fixed-order
// final block (deterministic fp64).  Gradient: pull per pin over its fanin and
// fanout rows (no atomics); pins with a wide fanout row get a warp each.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>

#include "device_common.cuh"
#include "internal.h"

namespace insta {

int ensure_fanout_words(DevGraph& g);   // clark.cu

struct TlParams {
  int32_t n;
  int64_t e;
  double lambda;
  const int32_t* __restrict__ fanin_ptr;
  const int32_t* __restrict__ fin_src;
  const int32_t* __restrict__ fin_arc;
  const int32_t* __restrict__ arc_sink;   // caller arc -> canonical sink
  const int32_t* __restrict__ order;      // canonical -> caller pin
  const int32_t* __restrict__ fo_ptr;
  const int32_t* __restrict__ fo_q;       // fanin position << 2 | unateness
  const int32_t* __restrict__ hv_list;    // wide-fanout pins (canonical)
  const int32_t* __restrict__ hv_of;
  int32_t num_wide;
  const float* __restrict__ x;            // caller order
  const float* __restrict__ y;
  const float* __restrict__ w;            // caller arc order
  double* partials;
  double* loss;
  float* gx;
  float* gy;
};

__device__ __forceinline__ double sgn(double d) { return d > 0.0 ? 1.0 : (d < 0.0 ? -1.0 : 0.0); }

constexpr int kTlThreads = 256;

__global__ void __launch_bounds__(kTlThreads) tl_loss_kernel(TlParams P) {
  __shared__ double s[kTlThreads];
  const long long q = blockIdx.x * (long long)kTlThreads + threadIdx.x;
  double v = 0.0;
  if (q < P.e) {
    const int arc = __ldg(P.fin_arc + q);
    const int f = __ldg(P.order + (__ldg(P.fin_src + q) & kSrcMask));
    const int t = __ldg(P.order + __ldg(P.arc_sink + arc));
    const double dx = double(__ldg(P.x + f)) - double(__ldg(P.x + t));
    const double dy = double(__ldg(P.y + f)) - double(__ldg(P.y + t));
    v = (fabs(dx) + fabs(dy)) * double(__ldg(P.w + arc));
  }
  s[threadIdx.x] = v;
  __syncthreads();
  for (int d = kTlThreads / 2; d > 0; d >>= 1) {
    if (threadIdx.x < d) s[threadIdx.x] += s[threadIdx.x + d];
    __syncthreads();
  }
  if (threadIdx.x == 0) P.partials[blockIdx.x] = s[0];
}

__global__ void __launch_bounds__(1024) tl_final_kernel(int nb, double lambda, const double* __restrict__ part,
                                                        double* loss) {
  __shared__ double s[1024];
  const int t = threadIdx.x, ch = (nb + 1023) / 1024;
  double v = 0.0;
  for (int b = t * ch; b < min(nb, (t + 1) * ch); ++b) v += part[b];
  s[t] = v;
  __syncthreads();
  for (int d = 512; d > 0; d >>= 1) {
    if (t < d) s[t] += s[t + d];
    __syncthreads();
  }
  if (t == 0) *loss = lambda * s[0];
}

// d/dx of the terms of pin i (canonical) over fanout entries k0, k0+step, ... (i = driver f)
__device__ __forceinline__ double2 tl_fanout(const TlParams& P, double xi, double yi, int k0, int k1, int step) {
  double gx = 0.0, gy = 0.0;
  for (int k = k0; k < k1; k += step) {
    const int q = int(uint32_t(__ldg(P.fo_q + k)) >> 2);
    const int arc = __ldg(P.fin_arc + q);
    const int t = __ldg(P.order + __ldg(P.arc_sink + arc));
    const double wk = double(__ldg(P.w + arc));
    gx += wk * sgn(xi - double(__ldg(P.x + t)));
    gy += wk * sgn(yi - double(__ldg(P.y + t)));
  }
  return make_double2(gx, gy);
}

// a thread per pin with a narrow fanout row: fanin terms (pin = sink t) + fanout terms (pin = driver f)
__global__ void tl_grad_kernel(TlParams P) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= P.n || __ldg(P.hv_of + p) >= 0) return;
  const int c = __ldg(P.order + p);
  const double xi = double(__ldg(P.x + c)), yi = double(__ldg(P.y + c));
  double gx = 0.0, gy = 0.0;
  for (int q = __ldg(P.fanin_ptr + p); q < __ldg(P.fanin_ptr + p + 1); ++q) {
    const int f = __ldg(P.order + (__ldg(P.fin_src + q) & kSrcMask));
    const double wk = double(__ldg(P.w + __ldg(P.fin_arc + q)));
    gx -= wk * sgn(double(__ldg(P.x + f)) - xi);
    gy -= wk * sgn(double(__ldg(P.y + f)) - yi);
  }
  const double2 o = tl_fanout(P, xi, yi, __ldg(P.fo_ptr + p), __ldg(P.fo_ptr + p + 1), 1);
  P.gx[c] = float(P.lambda * (gx + o.x));
  P.gy[c] = float(P.lambda * (gy + o.y));
}

// a warp per wide-fanout pin (lanes strided over the row, fixed shuffle tree)
__global__ void tl_grad_wide_kernel(TlParams P) {
  const long long h = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (h >= P.num_wide) return;
  const int p = __ldg(P.hv_list + h);
  const int c = __ldg(P.order + p);
  const double xi = double(__ldg(P.x + c)), yi = double(__ldg(P.y + c));
  double2 o = tl_fanout(P, xi, yi, __ldg(P.fo_ptr + p) + lane, __ldg(P.fo_ptr + p + 1), 32);
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) {
    o.x += __shfl_down_sync(0xffffffffu, o.x, d);
    o.y += __shfl_down_sync(0xffffffffu, o.y, d);
  }
  if (lane != 0) return;
  double gx = 0.0, gy = 0.0;
  for (int q = __ldg(P.fanin_ptr + p); q < __ldg(P.fanin_ptr + p + 1); ++q) {
    const int f = __ldg(P.order + (__ldg(P.fin_src + q) & kSrcMask));
    const double wk = double(__ldg(P.w + __ldg(P.fin_arc + q)));
    gx -= wk * sgn(double(__ldg(P.x + f)) - xi);
    gy -= wk * sgn(double(__ldg(P.y + f)) - yi);
  }
  P.gx[c] = float(P.lambda * (gx + o.x));
  P.gy[c] = float(P.lambda * (gy + o.y));
}

int launch_timing_loss(DevGraph& g, const float* x, const float* y, const float* w, float lambda_rc, double* loss,
                       float* gx, float* gy, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  int err = ensure_fanout_words(g);
  if (err) return err;
  const int nb = int((g.e + kTlThreads - 1) / kTlThreads);
  if (g.tl_cap < nb) {
    if (g.tl_partials) cudaFree(g.tl_partials);
    g.tl_partials = nullptr;
    cudaError_t e = cudaMalloc(&g.tl_partials, sizeof(double) * size_t(std::max(nb, 1)));
    if (e != cudaSuccess) return int(e);
    g.tl_cap = nb;
  }
  TlParams P{};
  P.n = g.n;
  P.e = g.e;
  P.lambda = double(lambda_rc);
  P.fanin_ptr = g.fanin_ptr;
  P.fin_src = g.fin_src;
  P.fin_arc = g.fin_arc;
  P.arc_sink = g.arc_sink;
  P.order = g.order;
  P.fo_ptr = g.cl_fo_ptr;
  P.fo_q = g.cl_fo_q;
  P.hv_list = g.cl_hv_list;
  P.hv_of = g.cl_hv_of;
  P.num_wide = g.cl_hv_ptr.empty() ? 0 : g.cl_hv_ptr.back();
  P.x = x;
  P.y = y;
  P.w = w;
  P.partials = g.tl_partials;
  P.loss = loss;
  P.gx = gx;
  P.gy = gy;
  if (loss) {
    if (nb > 0) {
      tl_loss_kernel<<<nb, kTlThreads, 0, st>>>(P);
      tl_final_kernel<<<1, 1024, 0, st>>>(nb, P.lambda, g.tl_partials, loss);
    } else {
      cudaMemsetAsync(loss, 0, sizeof(double), st);
    }
  }
  if (gx && gy && g.n > 0) {
    tl_grad_kernel<<<(g.n + 255) / 256, 256, 0, st>>>(P);
    if (P.num_wide > 0) tl_grad_wide_kernel<<<unsigned((32LL * P.num_wide + 255) / 256), 256, 0, st>>>(P);
  }
  return int(cudaGetLastError());
}

// Eq 8: lambda_2 = ||a|| / ||b|| (fixed-order fp64 sums of squares)
__global__ void __launch_bounds__(1024) norm_ratio_kernel(long long n, const float* __restrict__ a,
                                                          const float* __restrict__ b, double* out) {
  __shared__ double sa[1024], sb[1024];
  const int t = threadIdx.x;
  const long long ch = (n + 1023) / 1024;
  double va = 0.0, vb = 0.0;
  for (long long k = t * ch; k < min(n, (t + 1) * ch); ++k) {
    va += double(a[k]) * double(a[k]);
    vb += double(b[k]) * double(b[k]);
  }
  sa[t] = va;
  sb[t] = vb;
  __syncthreads();
  for (int d = 512; d > 0; d >>= 1) {
    if (t < d) {
      sa[t] += sa[t + d];
      sb[t] += sb[t + d];
    }
    __syncthreads();
  }
  if (t == 0) *out = sb[0] > 0.0 ? sqrt(sa[0]) / sqrt(sb[0]) : 0.0;
}

int launch_norm_ratio(int64_t n, const float* a, const float* b, double* out, void* stream) {
  norm_ratio_kernel<<<1, 1024, 0, static_cast<cudaStream_t>(stream)>>>(n, a, b, out);
  return int(cudaGetLastError());
}

}  // namespace insta
