// place.cu -- the device-side part of INSTA-Place:
// the timing objective of Eq 7,
//   L = lambda_RC * sum_k (|x_f - x_t| + |y_f - y_t|) * w_k,
// over every timing arc k = (f -> t) with a per-arc weight w_k (DESIGN.md
// R21: the arc's timing sensitivity, e.g. -(dTNS/dmean_R + dTNS/dmean_F) from
// insta_backward; 0 = not critical), its gradient w.r.t. the pin positions
// (subgradient sign(0) = 0), and the gradient-norm ratio of Eq 8.
//
// One pass, a thread per caller pin over its incident arcs (fanout then fanin,
// a CSR built once per graph in caller pin order): the pin's own position and
// row are read contiguously, each arc costs three 4-byte gathers (w_k and the
// other end's x, y).  Both ends of an arc take the same form,
//   d/dx_p  w |x_p - x_o| = w sign(x_p - x_o),
// so the gradient is one sum per pin (fixed order: deterministic, no atomics);
// the loss is summed at the arc's driver only.  Pins with a wide row get a
// warp each.  Loss: per-block fixed trees, then one fixed-order final block.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <vector>

#include "device_common.cuh"
#include "internal.h"

namespace insta {

constexpr int kPlWide = 64;        // incident arcs above which a pin gets a warp
constexpr int kTlThreads = 256;

struct TlParams {
  int32_t n;
  int32_t num_wide;
  int32_t nb;                             // thread-kernel blocks (partials [0, nb)), wide pins after
  double lambda;
  const int32_t* __restrict__ ptr;
  const int32_t* __restrict__ ent;
  const int32_t* __restrict__ arc;
  const int32_t* __restrict__ wide;
  const float* __restrict__ x;            // caller order
  const float* __restrict__ y;
  const float2* __restrict__ xy;          // (x, y) packed per pin (tl_pack_kernel): one 8-byte gather per arc end
  const float* __restrict__ w;            // caller arc order
  double* partials;
  float* gx;
  float* gy;
};

__device__ __forceinline__ double sgn(double d) { return d > 0.0 ? 1.0 : (d < 0.0 ? -1.0 : 0.0); }

// incident arcs k0, k0 + step, ... < k1 of pin (xi, yi): gradient sums and the driver-side loss.
// Four arcs per round: their row words, then their gathers, all in flight before any is used
// (the same sums in the same order as one arc at a time).
__device__ __forceinline__ void tl_row(const TlParams& P, double xi, double yi, int k0, int k1, int step,
                                       double& gx, double& gy, double& loss) {
  for (int k = k0; k < k1; k += 4 * step) {
    int32_t e[4], a[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int kk = k + j * step;
      e[j] = kk < k1 ? __ldg(P.ent + kk) : 0;
      a[j] = kk < k1 ? __ldg(P.arc + kk) : 0;
    }
    float2 po[4];
    float wv[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const bool v = k + j * step < k1;
      po[j] = v ? __ldg(P.xy + (e[j] & 0x7fffffff)) : make_float2(0.f, 0.f);
      wv[j] = v ? __ldg(P.w + a[j]) : 0.f;
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (k + j * step < k1) {
        const double wk = double(wv[j]);
        const double dx = xi - double(po[j].x), dy = yi - double(po[j].y);
        gx += wk * sgn(dx);
        gy += wk * sgn(dy);
        if (e[j] >= 0) loss += (fabs(dx) + fabs(dy)) * wk;   // counted once, at the driver
      }
    }
  }
}

__global__ void tl_pack_kernel(int n, const float* __restrict__ x, const float* __restrict__ y, float2* xy) {
  for (int p = blockIdx.x * blockDim.x + threadIdx.x; p < n; p += gridDim.x * blockDim.x)
    xy[p] = make_float2(__ldg(x + p), __ldg(y + p));
}

__device__ __forceinline__ double block_sum(double v, double* s) {
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0) s[w] = v;
  __syncthreads();
  double t = 0.0;
  if (threadIdx.x == 0)
    for (int k = 0; k < int(blockDim.x >> 5); ++k) t += s[k];
  return t;
}

__global__ void __launch_bounds__(kTlThreads) tl_pin_kernel(TlParams P, int want_grad) {
  __shared__ double s[kTlThreads / 32];
  const int p = blockIdx.x * kTlThreads + threadIdx.x;
  double loss = 0.0;
  if (p < P.n) {
    const int k0 = __ldg(P.ptr + p), k1 = __ldg(P.ptr + p + 1);
    if (k1 - k0 <= kPlWide) {
      const float2 pi = __ldg(P.xy + p);
      const double xi = double(pi.x), yi = double(pi.y);
      double gx = 0.0, gy = 0.0;
      tl_row(P, xi, yi, k0, k1, 1, gx, gy, loss);
      if (want_grad) {
        P.gx[p] = float(P.lambda * gx);
        P.gy[p] = float(P.lambda * gy);
      }
    }
  }
  const double t = block_sum(loss, s);
  if (threadIdx.x == 0) P.partials[blockIdx.x] = t;
}

// a warp per wide pin (lanes strided over the row, fixed shuffle tree)
__global__ void tl_wide_kernel(TlParams P, int want_grad) {
  const long long h = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (h >= P.num_wide) return;
  const int p = __ldg(P.wide + h);
  const double xi = double(__ldg(P.x + p)), yi = double(__ldg(P.y + p));
  double gx = 0.0, gy = 0.0, loss = 0.0;
  tl_row(P, xi, yi, __ldg(P.ptr + p) + lane, __ldg(P.ptr + p + 1), 32, gx, gy, loss);
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) {
    gx += __shfl_down_sync(0xffffffffu, gx, d);
    gy += __shfl_down_sync(0xffffffffu, gy, d);
    loss += __shfl_down_sync(0xffffffffu, loss, d);
  }
  if (lane != 0) return;
  if (want_grad) {
    P.gx[p] = float(P.lambda * gx);
    P.gy[p] = float(P.lambda * gy);
  }
  P.partials[P.nb + h] = loss;
}

__global__ void __launch_bounds__(1024) tl_final_kernel(int nb, double lambda, const double* __restrict__ part,
                                                        double* loss) {
  __shared__ double s[32];
  const int t = threadIdx.x, ch = (nb + 1023) / 1024;
  double v = 0.0;
  for (int b = t * ch; b < min(nb, (t + 1) * ch); ++b) v += part[b];
  const double r = block_sum(v, s);
  if (t == 0) *loss = lambda * r;
}

// incident-arc CSR in caller pin order (built once per graph from the host levelization)
static int ensure_place_csr(DevGraph& g) {
  if (g.num_pl_wide >= 0) return 0;
  const HostLevels& h = g.host;
  const int n = g.n;
  const int64_t E = g.e;
  if (2 * E >= (int64_t(1) << 31)) return int(cudaErrorInvalidValue);
  std::vector<int32_t> ptr(size_t(n) + 1, 0), ent(size_t(std::max<int64_t>(2 * E, 1))),
      arc(size_t(std::max<int64_t>(2 * E, 1))), afrom(size_t(std::max<int64_t>(E, 1))),
      ato(size_t(std::max<int64_t>(E, 1)));
  for (int k = 0; k < n; ++k) {   // canonical k: its fanin arcs end at order[k], its fanout arcs start there
    const int32_t p = h.order[size_t(k)];
    for (int32_t q = h.fanin_ptr[size_t(k)]; q < h.fanin_ptr[size_t(k) + 1]; ++q) ato[size_t(h.fanin_arc[size_t(q)])] = p;
    for (int32_t q = h.fanout_ptr[size_t(k)]; q < h.fanout_ptr[size_t(k) + 1]; ++q)
      afrom[size_t(h.fanout_arc[size_t(q)])] = p;
    ptr[size_t(p) + 1] = (h.fanin_ptr[size_t(k) + 1] - h.fanin_ptr[size_t(k)]) +
                         (h.fanout_ptr[size_t(k) + 1] - h.fanout_ptr[size_t(k)]);
  }
  for (int p = 0; p < n; ++p) ptr[size_t(p) + 1] += ptr[size_t(p)];
  std::vector<int32_t> fill(ptr.begin(), ptr.end() - 1);
  for (int64_t e = 0; e < E; ++e) {   // fanout entries first (ascending arc id), then fanin
    const int32_t f = afrom[size_t(e)];
    ent[size_t(fill[size_t(f)])] = ato[size_t(e)];
    arc[size_t(fill[size_t(f)]++)] = int32_t(e);
  }
  for (int64_t e = 0; e < E; ++e) {
    const int32_t t = ato[size_t(e)];
    ent[size_t(fill[size_t(t)])] = int32_t(uint32_t(afrom[size_t(e)]) | 0x80000000u);
    arc[size_t(fill[size_t(t)]++)] = int32_t(e);
  }
  std::vector<int32_t> wide;
  for (int p = 0; p < n; ++p)
    if (ptr[size_t(p) + 1] - ptr[size_t(p)] > kPlWide) wide.push_back(p);
  cudaError_t e = cudaMalloc(&g.pl_ptr, sizeof(int32_t) * ptr.size());
  if (e == cudaSuccess) e = cudaMalloc(&g.pl_ent, sizeof(int32_t) * ent.size());
  if (e == cudaSuccess) e = cudaMalloc(&g.pl_arc, sizeof(int32_t) * arc.size());
  if (e == cudaSuccess) e = cudaMalloc(&g.pl_wide, sizeof(int32_t) * std::max<size_t>(wide.size(), 1));
  if (e == cudaSuccess) e = cudaMemcpy(g.pl_ptr, ptr.data(), sizeof(int32_t) * ptr.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(g.pl_ent, ent.data(), sizeof(int32_t) * ent.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(g.pl_arc, arc.data(), sizeof(int32_t) * arc.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess && !wide.empty())
    e = cudaMemcpy(g.pl_wide, wide.data(), sizeof(int32_t) * wide.size(), cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return int(e);
  g.num_pl_wide = int32_t(wide.size());
  return 0;
}

int launch_timing_loss(DevGraph& g, const float* x, const float* y, const float* w, float lambda_rc, double* loss,
                       float* gx, float* gy, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  int err = ensure_place_csr(g);
  if (err) return err;
  const int nb = (g.n + kTlThreads - 1) / kTlThreads;
  const int np = nb + g.num_pl_wide;
  if (g.tl_cap < np) {
    if (g.tl_partials) cudaFree(g.tl_partials);
    g.tl_partials = nullptr;
    cudaError_t e = cudaMalloc(&g.tl_partials, sizeof(double) * size_t(std::max(np, 1)));
    if (e != cudaSuccess) return int(e);
    g.tl_cap = np;
  }
  TlParams P{};
  P.n = g.n;
  P.num_wide = g.num_pl_wide;
  P.nb = nb;
  P.lambda = double(lambda_rc);
  P.ptr = g.pl_ptr;
  P.ent = g.pl_ent;
  P.arc = g.pl_arc;
  P.wide = g.pl_wide;
  if (g.pl_xy_cap < g.n) {   // packed positions (scratch)
    if (g.pl_xy) cudaFree(g.pl_xy);
    g.pl_xy = nullptr;
    cudaError_t e = cudaMalloc(&g.pl_xy, sizeof(float2) * size_t(std::max(g.n, 1)));
    if (e != cudaSuccess) return int(e);
    g.pl_xy_cap = g.n;
  }
  P.x = x;
  P.y = y;
  P.xy = reinterpret_cast<const float2*>(g.pl_xy);
  P.w = w;
  P.partials = g.tl_partials;
  P.gx = gx;
  P.gy = gy;
  const int want_grad = gx && gy;
  if (!loss && !want_grad) return 0;
  if (np == 0) {
    if (loss) cudaMemsetAsync(loss, 0, sizeof(double), st);
    return int(cudaGetLastError());
  }
  if (g.n > 0)
    tl_pack_kernel<<<std::min((g.n + 255) / 256, 148 * 8), 256, 0, st>>>(g.n, x, y, reinterpret_cast<float2*>(g.pl_xy));
  if (nb > 0) tl_pin_kernel<<<nb, kTlThreads, 0, st>>>(P, want_grad);
  if (P.num_wide > 0) tl_wide_kernel<<<unsigned((32LL * P.num_wide + 255) / 256), 256, 0, st>>>(P, want_grad);
  if (loss) tl_final_kernel<<<1, 1024, 0, st>>>(np, P.lambda, g.tl_partials, loss);
  return int(cudaGetLastError());
}

// Eq 8: lambda_2 = ||a|| / ||b||.  Grid-wide: a fixed grid of kNrBlocks blocks,
// each thread sums squares over a fixed grid-stride set (coalesced float4 loads
// when aligned), fixed-order warp and block trees -> per-block partials; one
// block sums the partials in index order (deterministic fp64).
constexpr int kNrBlocks = 592, kNrThreads = 256;

__global__ void __launch_bounds__(kNrThreads) norm_partial_kernel(long long n, const float* __restrict__ a,
                                                                 const float* __restrict__ b, double* part) {
  __shared__ double s[kNrThreads / 32];
  double va = 0.0, vb = 0.0;
  const long long t = blockIdx.x * (long long)kNrThreads + threadIdx.x, stride = (long long)kNrBlocks * kNrThreads;
  const bool vec = ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b)) & 15) == 0;
  long long done = 0;
  if (vec) {
    const long long n4 = n / 4;
    const float4* a4 = reinterpret_cast<const float4*>(a);
    const float4* b4 = reinterpret_cast<const float4*>(b);
    for (long long k = t; k < n4; k += stride) {
      const float4 x = __ldg(a4 + k), y = __ldg(b4 + k);
      va += double(x.x) * double(x.x) + double(x.y) * double(x.y) + double(x.z) * double(x.z) + double(x.w) * double(x.w);
      vb += double(y.x) * double(y.x) + double(y.y) * double(y.y) + double(y.z) * double(y.z) + double(y.w) * double(y.w);
    }
    done = 4 * n4;
  }
  for (long long k = done + t; k < n; k += stride) {
    const double x = double(__ldg(a + k)), y = double(__ldg(b + k));
    va += x * x;
    vb += y * y;
  }
  const double ra = block_sum(va, s);
  __syncthreads();
  const double rb = block_sum(vb, s);
  if (threadIdx.x == 0) {
    part[2 * blockIdx.x] = ra;
    part[2 * blockIdx.x + 1] = rb;
  }
}

__global__ void __launch_bounds__(1024) norm_final_kernel(const double* __restrict__ part, double* out) {
  __shared__ double s[32];
  const int t = threadIdx.x;
  const double va = t < kNrBlocks ? part[2 * t] : 0.0, vb = t < kNrBlocks ? part[2 * t + 1] : 0.0;
  const double ra = block_sum(va, s);
  __syncthreads();
  const double rb = block_sum(vb, s);
  if (t == 0) *out = rb > 0.0 ? sqrt(ra) / sqrt(rb) : 0.0;
}

int launch_norm_ratio(int64_t n, const float* a, const float* b, double* out, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  double* part = nullptr;
  cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&part), sizeof(double) * 2 * kNrBlocks, st);
  if (e != cudaSuccess) return int(e);
  norm_partial_kernel<<<kNrBlocks, kNrThreads, 0, st>>>(n, a, b, part);
  norm_final_kernel<<<1, 1024, 0, st>>>(part, out);
  e = cudaGetLastError();
  const cudaError_t e2 = cudaFreeAsync(part, st);
  return int(e != cudaSuccess ? e : e2);
}

}  // namespace insta
