// kernels.cu -- sm_100a kernels of the INSTA hot path.
//
//  * forward: statistical arrival propagation, Eq 1-3 with the
//    Alg 1 / Alg 2 K = 1 merge (strict ">") or the LSE smooth max
//    of Eq 4.  Thread per pin (Alg 1 l.3 "outPinID"), both rf in one
//    pass, fanin rows read as one coalesced CSR slice (Alg 1 l.5-7).
//  * slack / WNS / TNS: deterministic two-level fp64 reduction.
//  * backward: Eq 6 softmax weights chained in reverse level order
//    (P:L152).  Pull-style: a pin's adjoint is the sum of the per-arc adjoints
//    its fanout sinks wrote (warp-cooperative segmented reduction over the
//    warp's concatenated fanout rows; no float atomics).  High-fanout drivers
//    (> kHeavy sinks) instead receive int64 fixed-point atomic adds from their
//    sinks (order-independent, hence still deterministic).
//
// Launch structure: the paper launches one kernel per timing
// level.  Here the default is ONE persistent cooperative kernel per
// pass: each CTA walks tiles of kTile consecutive canonical pins; before the
// pins of level l are computed the CTA waits on a device counter until every
// tile that intersects level l-1 has published (release/acquire), so the level
// barrier is a per-CTA wait, not a grid-wide sync, and topology loads for the
// next tile are issued before the wait.  schedule=1 keeps the per-level
// launch chain for comparison; both call the same __device__ pin functions
// with the same warp alignment, so they are bit-identical.
//
// Arithmetic: fp32, IEEE sqrt/div/exp/log, compiled with --fmad=false so that
// every kernel evaluates a candidate with the same rounding (bitwise
// reproducible; incremental == full).
#include <cuda_runtime.h>

#include <cfloat>
#include <cmath>
#include <algorithm>
#include <cstdint>

#include "internal.h"

namespace insta {

constexpr int kMaxF = 4;          // fanin arcs cached in registers per pin
constexpr int kHeavy = kHeavyFanout;  // fanout above which a driver uses atomic accumulation
constexpr int kHeavyBit = 29;     // fin_src bit: the source pin is a heavy driver
constexpr int32_t kSrcMask = (1 << kHeavyBit) - 1;
constexpr double kFix = 4294967296.0;  // 2^32 fixed-point scale of heavy accumulators

struct KParams {
  int32_t n, num_tiles, num_levels, num_src, num_ep;
  const int32_t* __restrict__ level_ptr;
  const int2* __restrict__ tile_lv;       // {first level, last level} of each tile
  const int32_t* __restrict__ level_ntiles;
  const int32_t* __restrict__ fanin_ptr;
  const int32_t* __restrict__ fin_src;
  const float4* __restrict__ fin_ms;
  const int32_t* __restrict__ fin_arc;
  const int32_t* __restrict__ fanout_ptr;
  const int32_t* __restrict__ fout;       // fanin position of each fanout entry
  const int32_t* __restrict__ heavy_slot; // [n] slot of heavy drivers, -1 otherwise
  const float4* __restrict__ src_ms;
  const int32_t* __restrict__ order;
  float4* state;
  float2* g;
  const float2* seed;
  unsigned long long* heavy_acc;          // [slots][2] fixed point
  uint32_t* done;                         // [L] per-level completion counters
  float* d_mean;
  float* d_src;
  float n_sigma, tau;
  uint32_t epoch;
};

// --------------------------------------------------------------------------
// memory-model helpers
// --------------------------------------------------------------------------
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Thread 0 of the CTA waits until level `l` has been published by all tiles
// that intersect it in pass `epoch`, then the CTA proceeds.
__device__ __forceinline__ void cta_wait_level(const KParams& P, int l) {
  if (threadIdx.x == 0) {
    const uint32_t target = P.epoch * uint32_t(P.level_ntiles[l]);
    if (ld_acquire(P.done + l) != target) {
      int ns = 20;
      while (ld_acquire(P.done + l) != target) {
        __nanosleep(ns);
        ns = ns < 160 ? ns * 2 : 160;
      }
    }
    __threadfence();
  }
  __syncthreads();
}

__device__ __forceinline__ void cta_publish_level(const KParams& P, int l) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(P.done + l, 1u);
  }
}

// --------------------------------------------------------------------------
// Eq 1-3 for one candidate.  st/ms layout {mu_R, mu_F, sig_R, sig_F}.
//   mu_c  = mu_j[s] + arc_mean[rf]                 (Eq 1, Alg 1 l.12)
//   sig_c = sqrt(sig_j[s]^2 + arc_std[rf]^2)       (Eq 2, Alg 1 l.13)
//   A_c   = mu_c + n_sigma * sig_c                 (Eq 3, Alg 1 l.14)
// --------------------------------------------------------------------------
struct Cand {
  float mu, sig, A;
};

__device__ __forceinline__ float comp_mu(const float4& v, int s) { return s ? v.y : v.x; }
__device__ __forceinline__ float comp_sig(const float4& v, int s) { return s ? v.w : v.z; }

__device__ __forceinline__ Cand make_cand(const float4& sj, const float4& ms, int rf, int s,
                                          float ns) {
  Cand c;
  const float sgj = comp_sig(sj, s), sge = comp_sig(ms, rf);
  c.mu = comp_mu(sj, s) + comp_mu(ms, rf);
  c.sig = sqrtf(sgj * sgj + sge * sge);
  c.A = c.mu + ns * c.sig;
  return c;
}

// number of source transitions of an arc for sink transition rf, and the k-th
// one: POS {rf}; NEG {~rf} (Alg 1 l.8); NON (rf, ~rf) (reading R3).
__device__ __forceinline__ int n_src_tr(int u) { return u == 2 ? 2 : 1; }
__device__ __forceinline__ int src_tr(int rf, int u, int k) { return (u == 1 || k == 1) ? (rf ^ 1) : rf; }

// Per-pin fanin view: the first kMaxF arcs live in registers, the rest are
// read from memory on demand (rare slow path for wide cells).
struct Fanin {
  int beg, nf;
  int32_t src[kMaxF];
  float4 ms[kMaxF];
  float4 st[kMaxF];
};

__device__ __forceinline__ void fanin_load_topology(const KParams& P, int i, Fanin& F) {
  F.beg = __ldg(P.fanin_ptr + i);
  F.nf = __ldg(P.fanin_ptr + i + 1) - F.beg;
#pragma unroll
  for (int k = 0; k < kMaxF; ++k) {
    if (k < F.nf) {
      F.src[k] = __ldg(P.fin_src + F.beg + k);
      F.ms[k] = __ldg(P.fin_ms + F.beg + k);
    }
  }
}

// Source states: written by this kernel in earlier levels, so read at L2 (.cg).
template <bool kVolatileState>
__device__ __forceinline__ void fanin_load_state(const KParams& P, Fanin& F) {
#pragma unroll
  for (int k = 0; k < kMaxF; ++k) {
    if (k < F.nf) {
      const float4* p = P.state + (F.src[k] & kSrcMask);
      F.st[k] = kVolatileState ? __ldcg(p) : __ldg(p);
    }
  }
}

template <bool kVolatileState, class Fn>
__device__ __forceinline__ void fanin_arc(const KParams& P, const Fanin& F, int k, Fn&& fn) {
  if (k < kMaxF) {
    fn(F.src[k], F.ms[k], F.st[k]);
  } else {
    const int32_t s = __ldg(P.fin_src + F.beg + k);
    const float4 ms = __ldg(P.fin_ms + F.beg + k);
    const float4* p = P.state + (s & kSrcMask);
    const float4 st = kVolatileState ? __ldcg(p) : __ldg(p);
    fn(s, ms, st);
  }
}

// Visit the candidates of (pin, rf) in canonical order: fanin row order, then
// source transition rf before ~rf.  fn(k, s, cand).
template <bool kVolatileState, class Fn>
__device__ __forceinline__ void for_each_cand(const KParams& P, const Fanin& F, int rf, Fn&& fn) {
  const float ns = P.n_sigma;
#pragma unroll
  for (int k = 0; k < kMaxF; ++k) {
    if (k < F.nf) {
      const int u = int(uint32_t(F.src[k]) >> kUnateShift);
      const int m = n_src_tr(u);
      for (int a = 0; a < m; ++a) {
        const int s = src_tr(rf, u, a);
        fn(k, s, make_cand(F.st[k], F.ms[k], rf, s, ns));
      }
    }
  }
  for (int k = kMaxF; k < F.nf; ++k) {
    fanin_arc<kVolatileState>(P, F, k, [&](int32_t srcw, const float4& ms, const float4& st) {
      const int u = int(uint32_t(srcw) >> kUnateShift);
      const int m = n_src_tr(u);
      for (int a = 0; a < m; ++a) {
        const int s = src_tr(rf, u, a);
        fn(k, s, make_cand(st, ms, rf, s, ns));
      }
    });
  }
}

// Merge result for one (pin, rf): first arg-max (strict ">") and, in LSE mode,
// the log-sum-exp normalizer S = sum exp((A_c - M)/tau).
struct Merge {
  float M, mu_best, sig_best, S;
  int k_best, s_best;
};

template <bool kLSE, bool kVolatileState>
__device__ __forceinline__ Merge merge_pin(const KParams& P, const Fanin& F, int rf) {
  Merge r;
  r.M = -INFINITY;
  r.mu_best = 0.f;
  r.sig_best = 0.f;
  r.k_best = -1;
  r.s_best = 0;
  r.S = 1.f;
  for_each_cand<kVolatileState>(P, F, rf, [&](int k, int s, const Cand& c) {
    if (r.k_best < 0 || c.A > r.M) {   // Alg 2 l.4: replace only if strictly greater
      r.M = c.A;
      r.mu_best = c.mu;
      r.sig_best = c.sig;
      r.k_best = k;
      r.s_best = s;
    }
  });
  if (kLSE) {
    float S = 0.f;
    const float tau = P.tau;
    const float M = r.M;
    for_each_cand<kVolatileState>(P, F, rf, [&](int, int, const Cand& c) { S += expf((c.A - M) / tau); });
    r.S = S;
  }
  return r;
}

// Forward for one non-source pin; returns the new state.
template <bool kLSE, bool kVolatileState>
__device__ __forceinline__ float4 forward_pin(const KParams& P, const Fanin& F) {
  float mu[2], sg[2];
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    const Merge m = merge_pin<kLSE, kVolatileState>(P, F, rf);
    sg[rf] = m.sig_best;
    if (kLSE) {
      // Eq 4: A_i = M + tau*log(sum exp((A_c - M)/tau)); reading R1: sigma_i =
      // sigma of the arg-max, mu_i = A_i - n_sigma*sigma_i.
      const float A = m.M + P.tau * logf(m.S);
      mu[rf] = A - P.n_sigma * m.sig_best;
    } else {
      mu[rf] = m.mu_best;   // Alg 1 l.15 / Alg 2 l.6 with K = 1
    }
  }
  return make_float4(mu[0], mu[1], sg[0], sg[1]);
}

__device__ __forceinline__ float4 source_state(const KParams& P, int i) {
  // P:L62 clock arrival of a startpoint: its (mean, std) per rf.
  return __ldg(P.src_ms + i);
}

// --------------------------------------------------------------------------
// Forward: persistent cooperative kernel
// --------------------------------------------------------------------------
__device__ __forceinline__ int pin_level(const KParams& P, int i, int lvl0) {
  int l = lvl0;
  while (__ldg(P.level_ptr + l + 1) <= i) ++l;
  return l;
}

template <bool kLSE>
__global__ void __launch_bounds__(kTile) fwd_persistent(KParams P) {
  for (int t = blockIdx.x; t < P.num_tiles; t += gridDim.x) {
    const int i = t * kTile + threadIdx.x;
    const bool valid = i < P.n;
    const int2 lv = __ldg(P.tile_lv + t);
    const int my_l = valid ? pin_level(P, i, lv.x) : -1;
    Fanin F;
    F.nf = 0;
    if (valid && my_l > 0) fanin_load_topology(P, i, F);   // issued before the wait
    for (int l = lv.x; l <= lv.y; ++l) {
      if (l > 0) cta_wait_level(P, l - 1);
      if (my_l == l) {
        if (l == 0) {
          P.state[i] = source_state(P, i);
        } else {
          fanin_load_state<true>(P, F);
          P.state[i] = forward_pin<kLSE, true>(P, F);
        }
      }
      cta_publish_level(P, l);
    }
  }
}

// One launch per level (schedule = 1): pins [lo, hi) of one level.
template <bool kLSE>
__global__ void __launch_bounds__(kTile) fwd_level(KParams P, int lo, int hi, int level) {
  const int i = lo + blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= hi) return;
  if (level == 0) {
    P.state[i] = source_state(P, i);
    return;
  }
  Fanin F;
  fanin_load_topology(P, i, F);
  fanin_load_state<false>(P, F);
  P.state[i] = forward_pin<kLSE, false>(P, F);
}

// --------------------------------------------------------------------------
// Backward
// --------------------------------------------------------------------------
// Warp-cooperative pull: lane's pin i in [seg_lo, seg_hi) owns fanout row
// [row_beg, row_end) (empty for inactive lanes and heavy drivers).  The warp
// walks the concatenated rows in chunks of 32 entries; each entry's owner is
// found by a shuffle binary search and summed by a segmented shuffle scan;
// segment tails accumulate into the owner lane.  Fixed order => deterministic.
__device__ __forceinline__ float2 warp_pull(const KParams& P, int row_beg, int row_end) {
  const unsigned full = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int r0 = __shfl_sync(full, row_beg, 0);
  const int r1 = __shfl_sync(full, row_end, 31);
  float ax = 0.f, ay = 0.f;
  for (int c = r0; c < r1; c += 32) {
    const int k = c + lane;
    // owner = last lane whose row_beg <= k (row_beg is non-decreasing over lanes)
    int o = 0;
#pragma unroll
    for (int step = 16; step >= 1; step >>= 1) {
      const int probe = o + step;
      const int rb = __shfl_sync(full, row_beg, probe);
      if (rb <= k) o = probe;
    }
    const int oend = __shfl_sync(full, row_end, o);
    const bool live = k < oend;   // also false for k >= r1 and inside skipped rows
    float vx = 0.f, vy = 0.f;
    if (live) {
      const float2 gv = __ldcg(P.g + __ldg(P.fout + k));
      vx = gv.x;
      vy = gv.y;
    }
    const int owner = live ? o : -1 - lane;   // dead entries are singleton segments
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const float tx = __shfl_up_sync(full, vx, d);
      const float ty = __shfl_up_sync(full, vy, d);
      const int to = __shfl_up_sync(full, owner, d);
      if (lane >= d && to == owner) {
        vx += tx;
        vy += ty;
      }
    }
    // each owner lane takes the inclusive-scan value at its last entry in this chunk
    const int lo = max(row_beg, c), hi = min(row_end, c + 32);
    const int tail = (hi - 1 - c) & 31;
    const float sx = __shfl_sync(full, vx, tail);
    const float sy = __shfl_sync(full, vy, tail);
    if (hi > lo) {
      ax += sx;
      ay += sy;
    }
  }
  return make_float2(ax, ay);
}

// Backward for one pin i at level l (>0 => has fanin) with adjoint abar of its
// corner arrival per rf (dL/dA_i = dL/dmu_i, reading R1).  Writes, for each
// fanin arc q, g[q] = per-source-transition adjoint and d_mean[arc] (Eq 6
// chain; hard mode: one-hot at the first arg-max).
template <bool kLSE>
__device__ __forceinline__ void backward_fanin(const KParams& P, int i, float2 abar) {
  Fanin F;
  fanin_load_topology(P, i, F);
  if (abar.x == 0.f && abar.y == 0.f) {
    for (int k = 0; k < F.nf; ++k) P.g[F.beg + k] = make_float2(0.f, 0.f);
    return;   // d_mean was zero-filled by the launcher
  }
  fanin_load_state<false>(P, F);
  float gs[kMaxF][2], gm[kMaxF][2];
#pragma unroll
  for (int k = 0; k < kMaxF; ++k) gs[k][0] = gs[k][1] = gm[k][0] = gm[k][1] = 0.f;
  const bool wide = F.nf > kMaxF;
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    const float ab = rf ? abar.y : abar.x;
    if (ab == 0.f) continue;
    const Merge m = merge_pin<kLSE, false>(P, F, rf);
    const float tau = P.tau, M = m.M, S = m.S;
    for_each_cand<false>(P, F, rf, [&](int k, int s, const Cand& c) {
      float w;
      if (kLSE) {
        w = expf((c.A - M) / tau) / S;                    // Eq 6
      } else {
        w = (k == m.k_best && s == m.s_best) ? 1.f : 0.f; // hard: one-hot at c*
      }
      const float a = w * ab;
      if (k < kMaxF) {
#pragma unroll
        for (int kk = 0; kk < kMaxF; ++kk) {
          if (kk == k) {
            gm[kk][rf] += a;
            gs[kk][s] += a;
          }
        }
      }
    });
    (void)wide;
  }
#pragma unroll
  for (int k = 0; k < kMaxF; ++k) {
    if (k < F.nf) {
      const int q = F.beg + k;
      P.g[q] = make_float2(gs[k][0], gs[k][1]);
      if (gm[k][0] != 0.f || gm[k][1] != 0.f)
        reinterpret_cast<float2*>(P.d_mean)[__ldg(P.fin_arc + q)] = make_float2(gm[k][0], gm[k][1]);
      if ((F.src[k] >> kHeavyBit) & 1) {
        const int slot = __ldg(P.heavy_slot + (F.src[k] & kSrcMask));
        if (gs[k][0] != 0.f)
          atomicAdd(P.heavy_acc + 2 * slot, (unsigned long long)__double2ll_rn(double(gs[k][0]) * kFix));
        if (gs[k][1] != 0.f)
          atomicAdd(P.heavy_acc + 2 * slot + 1, (unsigned long long)__double2ll_rn(double(gs[k][1]) * kFix));
      }
    }
  }
  // slow path: arcs beyond the register cache, one at a time
  for (int k = kMaxF; k < F.nf; ++k) {
    float ks[2] = {0.f, 0.f}, km[2] = {0.f, 0.f};
#pragma unroll
    for (int rf = 0; rf < 2; ++rf) {
      const float ab = rf ? abar.y : abar.x;
      if (ab == 0.f) continue;
      const Merge m = merge_pin<kLSE, false>(P, F, rf);
      const float tau = P.tau, M = m.M, S = m.S;
      for_each_cand<false>(P, F, rf, [&](int kc, int s, const Cand& c) {
        if (kc != k) return;
        const float w = kLSE ? expf((c.A - M) / tau) / S
                             : ((kc == m.k_best && s == m.s_best) ? 1.f : 0.f);
        const float a = w * ab;
        km[rf] += a;
        ks[s] += a;
      });
    }
    const int q = F.beg + k;
    const int32_t srcw = __ldg(P.fin_src + q);
    P.g[q] = make_float2(ks[0], ks[1]);
    if (km[0] != 0.f || km[1] != 0.f)
      reinterpret_cast<float2*>(P.d_mean)[__ldg(P.fin_arc + q)] = make_float2(km[0], km[1]);
    if ((srcw >> kHeavyBit) & 1) {
      const int slot = __ldg(P.heavy_slot + (srcw & kSrcMask));
      if (ks[0] != 0.f) atomicAdd(P.heavy_acc + 2 * slot, (unsigned long long)__double2ll_rn(double(ks[0]) * kFix));
      if (ks[1] != 0.f) atomicAdd(P.heavy_acc + 2 * slot + 1, (unsigned long long)__double2ll_rn(double(ks[1]) * kFix));
    }
  }
}

// Adjoint of pin i (seg_lo <= i < seg_hi are this warp's pins of the current
// level; lanes outside contribute empty rows): seed + pulled fanout sum, or
// the heavy accumulator for high-fanout drivers.
__device__ __forceinline__ float2 pin_adjoint(const KParams& P, int i, bool active, int seg_lo,
                                              int seg_hi) {
  const int ci = min(max(i, seg_lo), seg_hi);
  const int ci1 = min(max(i + 1, seg_lo), seg_hi);
  int rb = __ldg(P.fanout_ptr + ci);
  int re = __ldg(P.fanout_ptr + ci1);
  int slot = -1;
  if (active && re - rb > kHeavy) {
    slot = __ldg(P.heavy_slot + i);
    rb = re;   // skipped row (contributions arrive through the accumulator)
  }
  float2 a = warp_pull(P, rb, re);
  if (!active) return make_float2(0.f, 0.f);
  if (slot >= 0) {
    // all sinks are at deeper, completed levels: read and reset the accumulator
    unsigned long long* acc = P.heavy_acc + 2 * slot;
    const long long hx = (long long)atomicExch(acc, 0ull);
    const long long hy = (long long)atomicExch(acc + 1, 0ull);
    a.x = float(double(hx) / kFix);
    a.y = float(double(hy) / kFix);
  }
  const float2 sd = P.seed[i];
  return make_float2(sd.x + a.x, sd.y + a.y);
}

template <bool kLSE>
__device__ __forceinline__ void backward_pin(const KParams& P, int i, int l, float2 abar) {
  if (l == 0) {
    if (P.d_src) reinterpret_cast<float2*>(P.d_src)[__ldg(P.order + i)] = abar;
  } else {
    backward_fanin<kLSE>(P, i, abar);
  }
}

template <bool kLSE>
__global__ void __launch_bounds__(kTile) bwd_persistent(KParams P) {
  for (int r = blockIdx.x; r < P.num_tiles; r += gridDim.x) {
    const int t = P.num_tiles - 1 - r;
    const int base = t * kTile;
    const int i = base + threadIdx.x;
    const bool valid = i < P.n;
    const int2 lv = __ldg(P.tile_lv + t);
    const int my_l = valid ? pin_level(P, i, lv.x) : -1;
    const int wbase = base + (threadIdx.x & ~31);
    for (int l = lv.y; l >= lv.x; --l) {
      if (l + 1 < P.num_levels) cta_wait_level(P, l + 1);
      const int seg_lo = max(__ldg(P.level_ptr + l), wbase);
      const int seg_hi = max(min(__ldg(P.level_ptr + l + 1), wbase + 32), seg_lo);
      const bool active = my_l == l;
      const float2 abar = pin_adjoint(P, i, active, seg_lo, seg_hi);
      if (active) backward_pin<kLSE>(P, i, l, abar);
      cta_publish_level(P, l);
    }
  }
}

// One launch per level (schedule = 1).  Threads are aligned to global
// multiples of 32 pins so that warps see the same pins as in bwd_persistent.
template <bool kLSE>
__global__ void __launch_bounds__(kTile) bwd_level(KParams P, int lo, int hi, int level) {
  const int i = (lo & ~31) + blockIdx.x * blockDim.x + threadIdx.x;
  const int wbase = i & ~31;
  const int seg_lo = max(lo, wbase);
  const int seg_hi = max(min(hi, wbase + 32), seg_lo);
  const bool active = i >= lo && i < hi;
  if (wbase >= hi) return;   // whole warp outside the level
  const float2 abar = pin_adjoint(P, i, active, seg_lo, seg_hi);
  if (active) backward_pin<kLSE>(P, i, level, abar);
}

// Endpoint seeds: dL/dA_ep[rf*] = -dL/dslack (slack = RAT - A); TNS: dL/dslack
// = 1 where slack < 0.
__global__ void seed_kernel(int num_ep, const int32_t* __restrict__ ep_pin,
                            const float* __restrict__ slack, const uint8_t* __restrict__ rf_star,
                            const float* __restrict__ ep_seed, float2* seed) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= num_ep) return;
  const float d = ep_seed ? ep_seed[k] : (slack[k] < 0.f ? 1.f : 0.f);
  const float v = d == 0.f ? 0.f : -d;
  seed[ep_pin[k]] = rf_star[k] ? make_float2(0.f, v) : make_float2(v, 0.f);
}

// --------------------------------------------------------------------------
// Endpoint slack + WNS/TNS: slack = RAT - A, min over rf, tie -> R; TNS in
// fp64 with a fixed reduction tree (block partials, then the last block).
// --------------------------------------------------------------------------
constexpr int kRedThreads = 256;

__global__ void __launch_bounds__(kRedThreads)
slack_kernel(int num_ep, const int32_t* __restrict__ ep_pin, const float2* __restrict__ ep_rat,
             const float4* __restrict__ state, float n_sigma, float* slack, uint8_t* rf_star,
             double* partials, uint32_t* ticket, double* summary) {
  __shared__ double s_tns[kRedThreads];
  __shared__ double s_wns[kRedThreads];
  __shared__ double s_nv[kRedThreads];
  __shared__ bool s_last;
  const int k = blockIdx.x * kRedThreads + threadIdx.x;
  double tns = 0.0, wns = 0.0, nv = 0.0;
  if (k < num_ep) {
    const float4 st = __ldcg(state + ep_pin[k]);
    const float2 rat = ep_rat[k];
    const float aR = st.x + n_sigma * st.z;   // Eq 3
    const float aF = st.y + n_sigma * st.w;
    const float sR = rat.x - aR, sF = rat.y - aF;
    const bool fall = sF < sR;
    const float s = fall ? sF : sR;
    slack[k] = s;
    rf_star[k] = fall ? 1 : 0;
    if (s < 0.f) {
      tns = double(s);
      nv = 1.0;
    }
    wns = s < 0.f ? double(s) : 0.0;
  }
  s_tns[threadIdx.x] = tns;
  s_wns[threadIdx.x] = wns;
  s_nv[threadIdx.x] = nv;
  __syncthreads();
  for (int w = kRedThreads / 2; w > 0; w >>= 1) {
    if (threadIdx.x < w) {
      s_tns[threadIdx.x] += s_tns[threadIdx.x + w];
      s_wns[threadIdx.x] = fmin(s_wns[threadIdx.x], s_wns[threadIdx.x + w]);
      s_nv[threadIdx.x] += s_nv[threadIdx.x + w];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    partials[3 * blockIdx.x + 0] = s_tns[0];
    partials[3 * blockIdx.x + 1] = s_wns[0];
    partials[3 * blockIdx.x + 2] = s_nv[0];
    __threadfence();
    const uint32_t prev = atomicAdd(ticket, 1u);
    s_last = prev == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  tns = 0.0;
  wns = 0.0;
  nv = 0.0;
  for (int b = threadIdx.x; b < int(gridDim.x); b += kRedThreads) {
    tns += __ldcg(partials + 3 * b + 0);
    wns = fmin(wns, __ldcg(partials + 3 * b + 1));
    nv += __ldcg(partials + 3 * b + 2);
  }
  s_tns[threadIdx.x] = tns;
  s_wns[threadIdx.x] = wns;
  s_nv[threadIdx.x] = nv;
  __syncthreads();
  for (int w = kRedThreads / 2; w > 0; w >>= 1) {
    if (threadIdx.x < w) {
      s_tns[threadIdx.x] += s_tns[threadIdx.x + w];
      s_wns[threadIdx.x] = fmin(s_wns[threadIdx.x], s_wns[threadIdx.x + w]);
      s_nv[threadIdx.x] += s_nv[threadIdx.x + w];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    summary[0] = s_wns[0];
    summary[1] = s_tns[0];
    summary[2] = s_nv[0];
    *ticket = 0u;
  }
}

// --------------------------------------------------------------------------
// Small utility kernels
// --------------------------------------------------------------------------
__global__ void arrivals_kernel(int n, const float4* __restrict__ state,
                                const int32_t* __restrict__ order, float n_sigma, float2* A,
                                float2* mean, float2* sigma) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const float4 st = state[i];
  const int p = order[i];
  if (A) A[p] = make_float2(st.x + n_sigma * st.z, st.y + n_sigma * st.w);
  if (mean) mean[p] = make_float2(st.x, st.y);
  if (sigma) sigma[p] = make_float2(st.z, st.w);
}

__global__ void update_arcs_kernel(int64_t n, const int32_t* __restrict__ ids,
                                   const float2* __restrict__ mean,
                                   const float2* __restrict__ sigma,
                                   const int32_t* __restrict__ arc_pos, float4* fin_ms) {
  const int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (k >= n) return;
  const int q = arc_pos[ids[k]];
  const float2 m = mean[k], s = sigma[k];
  fin_ms[q] = make_float4(m.x, m.y, s.x, s.y);
}

// --------------------------------------------------------------------------
// Launchers
// --------------------------------------------------------------------------
static KParams make_params(DevGraph& g) {
  KParams P;
  P.n = g.n;
  P.num_tiles = g.num_tiles;
  P.num_levels = g.num_levels;
  P.num_src = g.num_src;
  P.num_ep = g.num_ep;
  P.level_ptr = g.level_ptr;
  P.tile_lv = g.tile_lv;
  P.level_ntiles = g.level_ntiles;
  P.fanin_ptr = g.fanin_ptr;
  P.fin_src = g.fin_src;
  P.fin_ms = g.fin_ms;
  P.fin_arc = g.fin_arc;
  P.fanout_ptr = g.fanout_ptr;
  P.fout = g.fout;
  P.heavy_slot = g.heavy_slot;
  P.src_ms = g.src_ms;
  P.order = g.order;
  P.state = g.state;
  P.g = g.g;
  P.seed = g.seed;
  P.heavy_acc = g.heavy_acc;
  P.done = nullptr;
  P.d_mean = nullptr;
  P.d_src = nullptr;
  P.n_sigma = 3.f;
  P.tau = 0.f;
  P.epoch = 0;
  return P;
}

template <class K>
static int occupancy(K kernel, int sms) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, kTile, 0);
  return b * sms;
}

int configure_grids(DevGraph& g) {
  int sms = 0, coop = 0;
  cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g.device);
  if (e != cudaSuccess) return int(e);
  cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, g.device);
  if (!coop) return int(cudaErrorNotSupported);
  int f = std::min(occupancy(fwd_persistent<false>, sms), occupancy(fwd_persistent<true>, sms));
  int b = std::min(occupancy(bwd_persistent<false>, sms), occupancy(bwd_persistent<true>, sms));
  if (f <= 0 || b <= 0) return int(cudaErrorLaunchOutOfResources);
  g.grid_fwd = std::max(1, std::min(f, g.num_tiles));
  g.grid_bwd = std::max(1, std::min(b, g.num_tiles));
  return int(cudaGetLastError());
}

static int coop_launch(const void* fn, int grid, KParams& P, cudaStream_t st) {
  void* args[] = {&P};
  return int(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kTile), args, 0, st));
}

// Level counters are never reset: pass e leaves done[l] == e * ntiles[l] (mod 2^32)
// and, within a pass, the counter only takes values (e-1)*ntiles[l] + j with
// j < ntiles[l], so modular equality with the target is exact across wrap-around.
static void bump_epoch(uint32_t& epoch) { ++epoch; }

int launch_slack(DevGraph& g, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (g.num_ep == 0) {
    return int(cudaMemsetAsync(g.summary, 0, sizeof(double) * 3, st));
  }
  const int blocks = (g.num_ep + kRedThreads - 1) / kRedThreads;
  slack_kernel<<<blocks, kRedThreads, 0, st>>>(g.num_ep, g.ep_pin, g.ep_rat, g.state,
                                              g.last_n_sigma, g.slack, g.rf_star, g.partials,
                                              g.ticket, g.summary);
  return int(cudaGetLastError());
}

int launch_forward(DevGraph& g, float n_sigma, float tau, int schedule, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  KParams P = make_params(g);
  P.n_sigma = n_sigma;
  P.tau = tau;
  const bool lse = tau > 0.f;
  int err = 0;
  if (g.n > 0) {
    if (schedule == 0) {
      bump_epoch(g.epoch_fwd);
      P.epoch = g.epoch_fwd;
      P.done = g.done_fwd;
      err = coop_launch(lse ? (const void*)fwd_persistent<true> : (const void*)fwd_persistent<false>,
                        g.grid_fwd, P, st);
    } else {
      const auto& lp = g.host.level_ptr;
      for (int l = 0; l < g.num_levels && !err; ++l) {
        const int lo = lp[l], hi = lp[l + 1];
        const int blocks = (hi - lo + kTile - 1) / kTile;
        if (lse) fwd_level<true><<<blocks, kTile, 0, st>>>(P, lo, hi, l);
        else fwd_level<false><<<blocks, kTile, 0, st>>>(P, lo, hi, l);
        err = int(cudaGetLastError());
      }
    }
  }
  if (err) return err;
  g.last_n_sigma = n_sigma;
  g.last_tau = tau;
  return launch_slack(g, stream);
}

int launch_backward(DevGraph& g, const float* ep_seed, float* d_arc_mean, float* d_src,
                    void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaMemsetAsync(d_arc_mean, 0, sizeof(float) * 2 * size_t(g.e), st);
  if (e != cudaSuccess) return int(e);
  if (d_src) {
    e = cudaMemsetAsync(d_src, 0, sizeof(float) * 2 * size_t(g.n), st);
    if (e != cudaSuccess) return int(e);
  }
  if (g.num_ep > 0) {
    seed_kernel<<<(g.num_ep + 255) / 256, 256, 0, st>>>(g.num_ep, g.ep_pin, g.slack, g.rf_star,
                                                        ep_seed, g.seed);
    int err = int(cudaGetLastError());
    if (err) return err;
  }
  if (g.n == 0) return 0;
  KParams P = make_params(g);
  P.n_sigma = g.last_n_sigma;
  P.tau = g.last_tau;
  P.d_mean = d_arc_mean;
  P.d_src = d_src;
  const bool lse = g.last_tau > 0.f;
  if (g.bwd_schedule == 0) {
    bump_epoch(g.epoch_bwd);
    P.epoch = g.epoch_bwd;
    P.done = g.done_bwd;
    return coop_launch(lse ? (const void*)bwd_persistent<true> : (const void*)bwd_persistent<false>,
                       g.grid_bwd, P, st);
  }
  const auto& lp = g.host.level_ptr;
  for (int l = g.num_levels - 1; l >= 0; --l) {
    const int lo = lp[l], hi = lp[l + 1];
    const int span = hi - (lo & ~31);
    const int blocks = (span + kTile - 1) / kTile;
    if (lse) bwd_level<true><<<blocks, kTile, 0, st>>>(P, lo, hi, l);
    else bwd_level<false><<<blocks, kTile, 0, st>>>(P, lo, hi, l);
    int err = int(cudaGetLastError());
    if (err) return err;
  }
  return 0;
}

int launch_update_arcs(DevGraph& g, int64_t n, const int32_t* ids, const float* mean,
                       const float* sigma, int incremental, void* stream) {
  (void)incremental;
  if (n <= 0) return 0;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int blocks = int((n + 255) / 256);
  update_arcs_kernel<<<blocks, 256, 0, st>>>(n, ids, reinterpret_cast<const float2*>(mean),
                                             reinterpret_cast<const float2*>(sigma), g.arc_pos,
                                             g.fin_ms);
  return int(cudaGetLastError());
}

int launch_forward_incremental(DevGraph& g, float n_sigma, float tau, void* stream) {
  return launch_forward(g, n_sigma, tau, 0, stream);
}

int launch_arrivals(DevGraph& g, float* A, float* mean, float* sigma, void* stream) {
  if (g.n == 0) return 0;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  arrivals_kernel<<<(g.n + 255) / 256, 256, 0, st>>>(
      g.n, g.state, g.order, g.last_n_sigma, reinterpret_cast<float2*>(A),
      reinterpret_cast<float2*>(mean), reinterpret_cast<float2*>(sigma));
  return int(cudaGetLastError());
}

int launch_copy_slack(DevGraph& g, float* slack, uint8_t* rf, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (g.num_ep == 0) return 0;
  if (slack) {
    cudaError_t e = cudaMemcpyAsync(slack, g.slack, sizeof(float) * g.num_ep,
                                    cudaMemcpyDeviceToDevice, st);
    if (e != cudaSuccess) return int(e);
  }
  if (rf) {
    cudaError_t e = cudaMemcpyAsync(rf, g.rf_star, g.num_ep, cudaMemcpyDeviceToDevice, st);
    if (e != cudaSuccess) return int(e);
  }
  return 0;
}

}  // namespace insta
