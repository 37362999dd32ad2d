// kernels.cu -- sm_100a kernels of the INSTA hot path.
//
//  * forward: statistical arrival propagation, Eq 1-3 with the
//    Alg 1 / Alg 2 K = 1 merge (strict ">") or the LSE smooth max
//    of Eq 4; both rf per pin in one pass (Alg 1 l.7).
//  * slack / WNS / TNS: deterministic two-level fp64 reduction.
//  * backward: Eq 6 softmax weights chained in reverse level order
//    (P:L152).  The forward stores what the backward needs (hard mode: the
//    arg-max candidate per pin and rf; LSE: the Eq 6 weights per fanin arc), so
//    the backward never re-reads arrival states.  A pin's adjoint is pulled
//    from the per-arc adjoints its fanout sinks wrote (no float atomics); very
//    high-fanout drivers (> kHeavyFanout sinks) instead receive int64
//    fixed-point atomic adds (order-independent, hence deterministic).
//
// Execution.  The paper launches one kernel per timing level
// (P:L113).  Here one persistent cooperative kernel per pass runs every level:
// each level is pre-cut into balanced contiguous pin chunks ("items"), one per
// resident CTA per round.  While a CTA works on item k, one thread has already
// issued TMA bulk copies (cp.async.bulk + mbarrier) that stage item k+1's CSR
// slice (row pointers, source ids, arc mean/sigma, weights) in shared memory.
// The level dependency is a per-level device counter: a CTA publishes level l
// with fence.acq_rel + red.relaxed after its last item of l, and waits with
// ld.acquire before its first item of l+1 -- no grid-wide barrier, and CTAs
// with no pins in a level never wait.  After the wait the only random accesses
// are the source-state gathers (forward) / per-arc adjoint gathers (backward),
// issued arc-parallel by all 1024 threads into shared memory.
//
// schedule = 1 launches the same item code once per level (no counters); both
// schedules are bit-identical.  Arithmetic: fp64 means, fp32 sigmas, IEEE
// sqrt/div/exp/log, --fmad=false: deterministic and bit-reproducible.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>

#include "internal.h"

namespace insta {

constexpr double kFix = 4294967296.0;  // 2^32: fixed-point scale of heavy accumulators

struct KParams {
  int32_t n, num_levels, grid;
  int32_t step_begin, step_end;  // item steps this launch runs
  int32_t wait;                  // 1 = persistent (level counters), 0 = per-level launch
  const int4* __restrict__ item_a;
  const int4* __restrict__ item_b;
  const int32_t* __restrict__ fanin_ptr;
  const int32_t* __restrict__ fin_src;
  const float4* __restrict__ fin_ms;
  const int32_t* __restrict__ fin_arc;
  const int32_t* __restrict__ lfo_ptr;
  const int32_t* __restrict__ lfo;
  const int32_t* __restrict__ heavy_slot;
  const float4* __restrict__ src_ms;
  const int32_t* __restrict__ order;
  PinState* state;
  int32_t* win;
  float4* wts;
  float2* g;
  const float2* seed;
  unsigned long long* heavy_acc;
  uint32_t* done;
  float* d_mean;
  float* d_src;
  float n_sigma, tau;
  uint32_t epoch;
};

// --------------------------------------------------------------------------
// PTX helpers: memory model, mbarrier, TMA bulk copy
// --------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void red_release(uint32_t* p) {
  asm volatile("fence.acq_rel.gpu;\n\tred.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(p) : "memory");
}

__device__ __forceinline__ void mbar_init(uint64_t* bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// 16-byte aligned window covering elements [a, b) of an array of esz-byte items
struct Window {
  int32_t off;     // element offset of a inside the window
  uint32_t bytes;  // bytes to copy
  int64_t start;   // first element copied
};

__device__ __forceinline__ Window window(int64_t a, int64_t b, int esz) {
  const int per = 16 / esz;
  Window w;
  w.start = a - (a % per);
  const int64_t end = ((b + per - 1) / per) * per;
  w.off = int32_t(a - w.start);
  w.bytes = b > a ? uint32_t((end - w.start) * esz) : 0u;
  return w;
}

// Level dependency: thread 0 spins on the counter, then the CTA proceeds.
__device__ __forceinline__ void wait_level(const KParams& P, int l) {
  if (threadIdx.x == 0) {
    const uint32_t target = P.epoch * uint32_t(P.grid);
    while (ld_acquire(P.done + l) != target) __nanosleep(20);
  }
  __syncthreads();
}

// --------------------------------------------------------------------------
// Eq 1-3 for one candidate: arc e = (j -> i), sink transition rf, source
// transition s.
//   mu_c  = mu_j[s] + arc_mean[rf]                 (Eq 1, Alg 1 l.12)
//   sig_c = sqrt(sig_j[s]^2 + arc_std[rf]^2)       (Eq 2, Alg 1 l.13)
//   A_c   = mu_c + n_sigma * sig_c                 (Eq 3, Alg 1 l.14)
// --------------------------------------------------------------------------
struct Gath {
  double mu0, mu1;
  float s0, s1;
};

struct Cand {
  double mu, A;
  float sig;
};

__device__ __forceinline__ Gath load_state_cg(const PinState* p) {
  const double2 m = __ldcg(reinterpret_cast<const double2*>(p));
  const float2 s = __ldcg(reinterpret_cast<const float2*>(p) + 2);
  Gath g;
  g.mu0 = m.x;
  g.mu1 = m.y;
  g.s0 = s.x;
  g.s1 = s.y;
  return g;
}

__device__ __forceinline__ Cand make_cand(const Gath& st, const float4& ms, int rf, int s, double ns) {
  const float sj = s ? st.s1 : st.s0;
  const float se = rf ? ms.w : ms.z;
  Cand c;
  c.mu = (s ? st.mu1 : st.mu0) + double(rf ? ms.y : ms.x);
  c.sig = sqrtf(sj * sj + se * se);
  c.A = c.mu + ns * double(c.sig);
  return c;
}

// source transitions of an arc for sink transition rf: POS {rf}; NEG {~rf}
// (Alg 1 l.8); NON (rf, ~rf) (reading R3).
__device__ __forceinline__ int n_src_tr(int u) { return u == 2 ? 2 : 1; }
__device__ __forceinline__ int src_tr(int rf, int u, int a) { return (u == 1 || a == 1) ? (rf ^ 1) : rf; }

// Forward of one non-source pin i with nf fanin arcs (first at fanin position
// q0); arc(k, srcw, ms, state) yields the k-th arc record and source state.
template <bool kLSE, class ArcFn>
__device__ __forceinline__ void fwd_pin(const KParams& P, int i, int nf, int q0, ArcFn&& arc) {
  const double ns = double(P.n_sigma);
  const double tau = double(P.tau);
  double mu_out[2], M[2];
  float sg_out[2], S[2];
  int win = 0;
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    double best = 0.0, bmu = 0.0;
    float bsg = 0.f;
    int bk = -1, bs = 0;
    for (int k = 0; k < nf; ++k) {
      int32_t w;
      float4 ms;
      Gath st;
      arc(k, w, ms, st);
      const int u = int(uint32_t(w) >> kUnateShift);
      for (int a = 0; a < n_src_tr(u); ++a) {
        const int s = src_tr(rf, u, a);
        const Cand c = make_cand(st, ms, rf, s, ns);
        if (bk < 0 || c.A > best) {   // Alg 2 l.4: replace only if strictly greater
          best = c.A;
          bmu = c.mu;
          bsg = c.sig;
          bk = k;
          bs = s;
        }
      }
    }
    M[rf] = best;
    sg_out[rf] = bsg;
    win |= (bk | (bs << 15)) << (16 * rf);
    if (kLSE) {
      // Eq 4: A_i = M + tau * log(sum_c exp((A_c - M) / tau)); reading R1:
      // sigma_i = sigma of the arg-max, mu_i = A_i - n_sigma * sigma_i.
      float sum = 0.f;
      for (int k = 0; k < nf; ++k) {
        int32_t w;
        float4 ms;
        Gath st;
        arc(k, w, ms, st);
        const int u = int(uint32_t(w) >> kUnateShift);
        for (int a = 0; a < n_src_tr(u); ++a) {
          const Cand c = make_cand(st, ms, rf, src_tr(rf, u, a), ns);
          sum += expf(float((c.A - best) / tau));
        }
      }
      S[rf] = sum;
      mu_out[rf] = (best + tau * double(logf(sum))) - ns * double(bsg);
    } else {
      mu_out[rf] = bmu;   // Alg 1 l.15 / Alg 2 l.6 with K = 1
    }
  }
  PinState* o = P.state + i;
  reinterpret_cast<double2*>(o)[0] = make_double2(mu_out[0], mu_out[1]);
  reinterpret_cast<float4*>(o)[1] = make_float4(sg_out[0], sg_out[1], 0.f, 0.f);
  if (!kLSE) {
    P.win[i] = win;
  } else {
    // Eq 6 weights w[rf][s] of every candidate, stored per fanin arc
    for (int k = 0; k < nf; ++k) {
      int32_t w;
      float4 ms;
      Gath st;
      arc(k, w, ms, st);
      const int u = int(uint32_t(w) >> kUnateShift);
      float wt[2][2] = {{0.f, 0.f}, {0.f, 0.f}};
#pragma unroll
      for (int rf = 0; rf < 2; ++rf) {
        for (int a = 0; a < n_src_tr(u); ++a) {
          const int s = src_tr(rf, u, a);
          const Cand c = make_cand(st, ms, rf, s, ns);
          wt[rf][s] = expf(float((c.A - M[rf]) / tau)) / S[rf];
        }
      }
      P.wts[q0 + k] = make_float4(wt[0][0], wt[0][1], wt[1][0], wt[1][1]);
    }
  }
}

// --------------------------------------------------------------------------
// Forward kernel
// --------------------------------------------------------------------------
struct FwdStage {
  int32_t ptr[kFwdPins + 8];
  int32_t src[kFwdArcs + 8];
  float4 ms[kFwdArcs];
};
constexpr size_t kFwdSmem = 2 * sizeof(FwdStage) + sizeof(Gath) * kFwdArcs;

__device__ __forceinline__ bool fwd_staged(const int4& A, const int4& B) {
  return A.y > A.x && B.x > 0 && !(B.y & kItemDirect);
}

// thread 0: issue the bulk copies staging item (step, c) into `st`
__device__ __forceinline__ void fwd_prefetch(const KParams& P, FwdStage* st, uint64_t* bar, int step,
                                             int c) {
  const int4 A = __ldg(P.item_a + size_t(step) * P.grid + c);
  const int4 B = __ldg(P.item_b + size_t(step) * P.grid + c);
  if (!fwd_staged(A, B)) return;
  const Window wp = window(A.x, A.y + 1, 4);
  const Window ws = window(A.z, A.w, 4);
  const uint32_t bms = uint32_t(A.w - A.z) * 16u;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_expect_tx(bar, wp.bytes + ws.bytes + bms);
  bulk_g2s(st->ptr, P.fanin_ptr + wp.start, wp.bytes, bar);
  if (ws.bytes) bulk_g2s(st->src, P.fin_src + ws.start, ws.bytes, bar);
  if (bms) bulk_g2s(st->ms, P.fin_ms + A.z, bms, bar);
}

template <bool kLSE>
__global__ void __launch_bounds__(kThreads, 1) fwd_kernel(KParams P) {
  extern __shared__ __align__(128) unsigned char smem[];
  FwdStage* stage = reinterpret_cast<FwdStage*>(smem);
  Gath* gath = reinterpret_cast<Gath*>(smem + 2 * sizeof(FwdStage));
  __shared__ __align__(8) uint64_t bar[2];
  const int c = blockIdx.x;
  const int tid = threadIdx.x;
  if (tid == 0) {
    mbar_init(&bar[0]);
    mbar_init(&bar[1]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  uint32_t phase0 = 0, phase1 = 0;
  int waited = -1;
  if (tid == 0 && P.step_begin < P.step_end) fwd_prefetch(P, &stage[0], &bar[0], P.step_begin, c);
  for (int k = P.step_begin; k < P.step_end; ++k) {
    const int buf = (k - P.step_begin) & 1;
    const int4 A = __ldg(P.item_a + size_t(k) * P.grid + c);   // {pin_lo, pin_hi, arc_lo, arc_hi}
    const int4 B = __ldg(P.item_b + size_t(k) * P.grid + c);   // {level, flags}
    const int l = B.x;
    if (tid == 0 && k + 1 < P.step_end) fwd_prefetch(P, &stage[buf ^ 1], &bar[buf ^ 1], k + 1, c);
    if (A.y > A.x) {
      if (l == 0) {
        // startpoints: clock arrival distribution, mean and std per rf
        for (int i = A.x + tid; i < A.y; i += kThreads) {
          const float4 s = __ldg(P.src_ms + i);
          PinState* o = P.state + i;
          reinterpret_cast<double2*>(o)[0] = make_double2(double(s.x), double(s.y));
          reinterpret_cast<float4*>(o)[1] = make_float4(s.z, s.w, 0.f, 0.f);
        }
      } else if (!(B.y & kItemDirect)) {
        if (buf == 0) {
          mbar_wait(&bar[0], phase0);
          phase0 ^= 1;
        } else {
          mbar_wait(&bar[1], phase1);
          phase1 ^= 1;
        }
        if (P.wait && waited != l) {
          wait_level(P, l - 1);
          waited = l;
        }
        const FwdStage& S = stage[buf];
        const int po = A.x & 3, so = A.z & 3;
        const int na = A.w - A.z;
        for (int a = tid; a < na; a += kThreads)
          gath[a] = load_state_cg(P.state + (S.src[so + a] & kSrcMask));
        __syncthreads();
        for (int p = tid; p < A.y - A.x; p += kThreads) {
          const int b0 = S.ptr[po + p] - A.z;
          const int b1 = S.ptr[po + p + 1] - A.z;
          fwd_pin<kLSE>(P, A.x + p, b1 - b0, A.z + b0,
                        [&](int kk, int32_t& w, float4& ms, Gath& st) {
                          w = S.src[so + b0 + kk];
                          ms = S.ms[b0 + kk];
                          st = gath[b0 + kk];
                        });
        }
      } else {
        if (P.wait && waited != l) {
          wait_level(P, l - 1);
          waited = l;
        }
        for (int i = A.x + tid; i < A.y; i += kThreads) {
          const int b0 = __ldg(P.fanin_ptr + i), b1 = __ldg(P.fanin_ptr + i + 1);
          fwd_pin<kLSE>(P, i, b1 - b0, b0, [&](int kk, int32_t& w, float4& ms, Gath& st) {
            w = __ldg(P.fin_src + b0 + kk);
            ms = __ldg(P.fin_ms + b0 + kk);
            st = load_state_cg(P.state + (w & kSrcMask));
          });
        }
      }
    }
    __syncthreads();
    if ((B.y & kItemLast) && P.wait && tid == 0) red_release(P.done + l);
  }
}

// --------------------------------------------------------------------------
// Backward kernel
// --------------------------------------------------------------------------
struct BwdStage {
  int32_t lptr[kBwdPins + 8];   // light fanout row pointers
  int32_t lfo[kBwdFanout + 8];  // fanin position of each light fanout entry
  int32_t fptr[kBwdPins + 8];   // fanin row pointers
  int32_t src[kBwdArcs + 8];    // fin_src
  int32_t arc[kBwdArcs + 8];    // caller arc ids
  int32_t win[kBwdPins + 8];    // hard-mode winners
  float2 seed[kBwdPins + 8];
  float4 wts[kBwdArcs];         // LSE weights
};
constexpr size_t kBwdSmem = 2 * sizeof(BwdStage) + sizeof(float2) * kBwdFanout;

__device__ __forceinline__ bool bwd_staged(const int4& A, const int4& B) {
  return A.y > A.x && !(B.w & kItemDirect);
}

template <bool kLSE>
__device__ __forceinline__ void bwd_prefetch(const KParams& P, BwdStage* st, uint64_t* bar, int step,
                                             int c) {
  const int4 A = __ldg(P.item_a + size_t(step) * P.grid + c);   // {pin_lo, pin_hi, lfo_lo, lfo_hi}
  const int4 B = __ldg(P.item_b + size_t(step) * P.grid + c);   // {arc_lo, arc_hi, level, flags}
  if (!bwd_staged(A, B)) return;
  const Window wl = window(A.x, A.y + 1, 4);   // lfo_ptr and fanin_ptr: same pin window
  const Window wf = window(A.z, A.w, 4);
  const Window wa = window(B.x, B.y, 4);
  const Window wsd = window(A.x, A.y, 8);
  const Window ww = window(A.x, A.y, 4);
  const uint32_t bw = kLSE ? uint32_t(B.y - B.x) * 16u : 0u;
  const uint32_t total = 2 * wl.bytes + wf.bytes + 2 * wa.bytes + wsd.bytes + (kLSE ? bw : ww.bytes);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_expect_tx(bar, total);
  bulk_g2s(st->lptr, P.lfo_ptr + wl.start, wl.bytes, bar);
  if (wf.bytes) bulk_g2s(st->lfo, P.lfo + wf.start, wf.bytes, bar);
  bulk_g2s(st->fptr, P.fanin_ptr + wl.start, wl.bytes, bar);
  if (wa.bytes) {
    bulk_g2s(st->src, P.fin_src + wa.start, wa.bytes, bar);
    bulk_g2s(st->arc, P.fin_arc + wa.start, wa.bytes, bar);
  }
  bulk_g2s(st->seed, P.seed + wsd.start, wsd.bytes, bar);
  if (kLSE) {
    if (bw) bulk_g2s(st->wts, P.wts + B.x, bw, bar);
  } else {
    bulk_g2s(st->win, P.win + ww.start, ww.bytes, bar);
  }
}

__device__ __forceinline__ void heavy_add(const KParams& P, int32_t srcw, float gx, float gy) {
  if (!((srcw >> kHeavyBit) & 1)) return;
  const int slot = __ldg(P.heavy_slot + (srcw & kSrcMask));
  if (gx != 0.f) atomicAdd(P.heavy_acc + 2 * slot, (unsigned long long)__double2ll_rn(double(gx) * kFix));
  if (gy != 0.f) atomicAdd(P.heavy_acc + 2 * slot + 1, (unsigned long long)__double2ll_rn(double(gy) * kFix));
}

// Sink side of a pin (nf fanin arcs from fanin position q0) with adjoint ab:
// per arc, g = adjoint to the source's {R, F} and dL/d(arc mean) (Eq 6 chain;
// hard mode: one-hot at the recorded arg-max).
template <bool kLSE, class ArcFn>
__device__ __forceinline__ void bwd_sink(const KParams& P, int nf, int q0, float2 ab, int32_t win,
                                         ArcFn&& arc) {
  const float abr[2] = {ab.x, ab.y};
  for (int k = 0; k < nf; ++k) {
    int32_t srcw, arcid;
    float4 w4;
    arc(k, srcw, arcid, w4);
    float w[2][2];
    if (kLSE) {
      w[0][0] = w4.x;
      w[0][1] = w4.y;
      w[1][0] = w4.z;
      w[1][1] = w4.w;
    } else {
#pragma unroll
      for (int rf = 0; rf < 2; ++rf) {
        const int wv = (win >> (16 * rf)) & 0xffff;
        const bool hit = (wv & 0x7fff) == k;
        w[rf][0] = (hit && (wv >> 15) == 0) ? 1.f : 0.f;
        w[rf][1] = (hit && (wv >> 15) == 1) ? 1.f : 0.f;
      }
    }
    float gm[2], gs[2] = {0.f, 0.f};
#pragma unroll
    for (int rf = 0; rf < 2; ++rf) {
      const float a0 = w[rf][0] * abr[rf], a1 = w[rf][1] * abr[rf];
      gm[rf] = a0 + a1;
      gs[0] += a0;
      gs[1] += a1;
    }
    P.g[q0 + k] = make_float2(gs[0], gs[1]);
    if (gm[0] != 0.f || gm[1] != 0.f)
      reinterpret_cast<float2*>(P.d_mean)[arcid] = make_float2(gm[0], gm[1]);
    heavy_add(P, srcw, gs[0], gs[1]);
  }
}

__device__ __forceinline__ float2 heavy_take(const KParams& P, int i) {
  const int slot = __ldg(P.heavy_slot + i);
  if (slot < 0) return make_float2(0.f, 0.f);
  // every sink of i is at a deeper, completed level: read and reset
  const long long hx = (long long)atomicExch(P.heavy_acc + 2 * slot, 0ull);
  const long long hy = (long long)atomicExch(P.heavy_acc + 2 * slot + 1, 0ull);
  return make_float2(float(double(hx) / kFix), float(double(hy) / kFix));
}

template <bool kLSE>
__global__ void __launch_bounds__(kThreads, 1) bwd_kernel(KParams P) {
  extern __shared__ __align__(128) unsigned char smem[];
  BwdStage* stage = reinterpret_cast<BwdStage*>(smem);
  float2* gg = reinterpret_cast<float2*>(smem + 2 * sizeof(BwdStage));
  __shared__ __align__(8) uint64_t bar[2];
  const int c = blockIdx.x;
  const int tid = threadIdx.x;
  if (tid == 0) {
    mbar_init(&bar[0]);
    mbar_init(&bar[1]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  uint32_t phase0 = 0, phase1 = 0;
  int waited = -1;
  if (tid == 0 && P.step_begin < P.step_end) bwd_prefetch<kLSE>(P, &stage[0], &bar[0], P.step_begin, c);
  for (int k = P.step_begin; k < P.step_end; ++k) {
    const int buf = (k - P.step_begin) & 1;
    const int4 A = __ldg(P.item_a + size_t(k) * P.grid + c);   // {pin_lo, pin_hi, lfo_lo, lfo_hi}
    const int4 B = __ldg(P.item_b + size_t(k) * P.grid + c);   // {arc_lo, arc_hi, level, flags}
    const int l = B.z;
    if (tid == 0 && k + 1 < P.step_end) bwd_prefetch<kLSE>(P, &stage[buf ^ 1], &bar[buf ^ 1], k + 1, c);
    if (A.y > A.x) {
      const bool wait_needed = P.wait && l + 1 < P.num_levels && waited != l;
      if (!(B.w & kItemDirect)) {
        if (buf == 0) {
          mbar_wait(&bar[0], phase0);
          phase0 ^= 1;
        } else {
          mbar_wait(&bar[1], phase1);
          phase1 ^= 1;
        }
        if (wait_needed) {
          wait_level(P, l + 1);
          waited = l;
        }
        const BwdStage& S = stage[buf];
        const int lo = A.x & 3, fo = A.z & 3, ao = B.x & 3, so = A.x & 1;
        const int nfo = A.w - A.z;
        for (int e = tid; e < nfo; e += kThreads) gg[e] = __ldcg(P.g + S.lfo[fo + e]);
        __syncthreads();
        for (int p = tid; p < A.y - A.x; p += kThreads) {
          const int i = A.x + p;
          // pull: seed + sum of the sinks' per-arc adjoints (+ heavy accumulator)
          const int r0 = S.lptr[lo + p] - A.z, r1 = S.lptr[lo + p + 1] - A.z;
          float2 ab = S.seed[so + p];
          float sx = 0.f, sy = 0.f;
          for (int r = r0; r < r1; ++r) {
            sx += gg[r].x;
            sy += gg[r].y;
          }
          const float2 h = heavy_take(P, i);
          ab.x += sx + h.x;
          ab.y += sy + h.y;
          if (l == 0) {
            if (P.d_src) reinterpret_cast<float2*>(P.d_src)[__ldg(P.order + i)] = ab;
          } else {
            const int b0 = S.fptr[lo + p] - B.x, b1 = S.fptr[lo + p + 1] - B.x;
            bwd_sink<kLSE>(P, b1 - b0, B.x + b0, ab, S.win[lo + p],
                           [&](int kk, int32_t& srcw, int32_t& arcid, float4& w4) {
                             srcw = S.src[ao + b0 + kk];
                             arcid = S.arc[ao + b0 + kk];
                             if (kLSE) w4 = S.wts[b0 + kk];
                           });
          }
        }
      } else {
        if (wait_needed) {
          wait_level(P, l + 1);
          waited = l;
        }
        for (int i = A.x + tid; i < A.y; i += kThreads) {
          float2 ab = P.seed[i];
          float sx = 0.f, sy = 0.f;
          const int r0 = __ldg(P.lfo_ptr + i), r1 = __ldg(P.lfo_ptr + i + 1);
          for (int r = r0; r < r1; ++r) {
            const float2 v = __ldcg(P.g + __ldg(P.lfo + r));
            sx += v.x;
            sy += v.y;
          }
          const float2 h = heavy_take(P, i);
          ab.x += sx + h.x;
          ab.y += sy + h.y;
          if (l == 0) {
            if (P.d_src) reinterpret_cast<float2*>(P.d_src)[__ldg(P.order + i)] = ab;
          } else {
            const int b0 = __ldg(P.fanin_ptr + i), b1 = __ldg(P.fanin_ptr + i + 1);
            bwd_sink<kLSE>(P, b1 - b0, b0, ab, kLSE ? 0 : P.win[i],
                           [&](int kk, int32_t& srcw, int32_t& arcid, float4& w4) {
                             srcw = __ldg(P.fin_src + b0 + kk);
                             arcid = __ldg(P.fin_arc + b0 + kk);
                             if (kLSE) w4 = P.wts[b0 + kk];
                           });
          }
        }
      }
    }
    __syncthreads();
    if ((B.w & kItemLast) && P.wait && tid == 0) red_release(P.done + l);
  }
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
             const PinState* __restrict__ state, float n_sigma, float* slack, uint8_t* rf_star,
             double* partials, uint32_t* ticket, double* summary) {
  __shared__ double s_tns[kRedThreads];
  __shared__ double s_wns[kRedThreads];
  __shared__ double s_nv[kRedThreads];
  __shared__ bool s_last;
  const int k = blockIdx.x * kRedThreads + threadIdx.x;
  double tns = 0.0, wns = 0.0, nv = 0.0;
  if (k < num_ep) {
    const Gath st = load_state_cg(state + ep_pin[k]);
    const float2 rat = ep_rat[k];
    const double ns = double(n_sigma);
    const double sR = double(rat.x) - (st.mu0 + ns * double(st.s0));   // Eq 3 corner
    const double sF = double(rat.y) - (st.mu1 + ns * double(st.s1));
    const bool fall = sF < sR;
    const double s = fall ? sF : sR;
    slack[k] = float(s);
    rf_star[k] = fall ? 1 : 0;
    if (s < 0.0) {
      tns = s;
      nv = 1.0;
      wns = s;
    }
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
__global__ void arrivals_kernel(int n, const PinState* __restrict__ state,
                                const int32_t* __restrict__ order, float n_sigma, float2* A,
                                float2* mean, float2* sigma) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const Gath st = load_state_cg(state + i);
  const int p = order[i];
  const double ns = double(n_sigma);
  if (A) A[p] = make_float2(float(st.mu0 + ns * double(st.s0)), float(st.mu1 + ns * double(st.s1)));
  if (mean) mean[p] = make_float2(float(st.mu0), float(st.mu1));
  if (sigma) sigma[p] = make_float2(st.s0, st.s1);
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
static KParams make_params(DevGraph& g, bool bwd) {
  KParams P{};
  P.n = g.n;
  P.num_levels = g.num_levels;
  P.grid = g.grid;
  P.item_a = bwd ? g.bwd_a : g.fwd_a;
  P.item_b = bwd ? g.bwd_b : g.fwd_b;
  P.fanin_ptr = g.fanin_ptr;
  P.fin_src = g.fin_src;
  P.fin_ms = g.fin_ms;
  P.fin_arc = g.fin_arc;
  P.lfo_ptr = g.lfo_ptr;
  P.lfo = g.lfo;
  P.heavy_slot = g.heavy_slot;
  P.src_ms = g.src_ms;
  P.order = g.order;
  P.state = g.state;
  P.win = g.win;
  P.wts = g.wts;
  P.g = g.g;
  P.seed = g.seed;
  P.heavy_acc = g.heavy_acc;
  P.done = bwd ? g.done_bwd : g.done_fwd;
  P.n_sigma = 3.f;
  P.tau = 0.f;
  return P;
}

template <class K>
static int set_smem(K kernel, size_t bytes) {
  return int(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bytes)));
}

int query_grid(int device, int* grid) {
  int sms = 0, coop = 0;
  cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) return int(e);
  cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, device);
  if (!coop) return int(cudaErrorNotSupported);
  int err = set_smem(fwd_kernel<false>, kFwdSmem);
  if (!err) err = set_smem(fwd_kernel<true>, kFwdSmem);
  if (!err) err = set_smem(bwd_kernel<false>, kBwdSmem);
  if (!err) err = set_smem(bwd_kernel<true>, kBwdSmem);
  if (err) return err;
  int occ = 1 << 30, b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, fwd_kernel<false>, kThreads, kFwdSmem);
  occ = std::min(occ, b);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, fwd_kernel<true>, kThreads, kFwdSmem);
  occ = std::min(occ, b);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, bwd_kernel<false>, kThreads, kBwdSmem);
  occ = std::min(occ, b);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, bwd_kernel<true>, kThreads, kBwdSmem);
  occ = std::min(occ, b);
  if (occ <= 0) return int(cudaErrorLaunchOutOfResources);
  *grid = occ * sms;
  return int(cudaGetLastError());
}

static int launch_items(const void* fn, size_t smem, KParams& P, const ItemTable& T, bool bwd,
                        int schedule, cudaStream_t st) {
  if (schedule == 0) {
    P.wait = 1;
    P.step_begin = 0;
    P.step_end = T.num_steps;
    void* args[] = {&P};
    return int(cudaLaunchCooperativeKernel(fn, dim3(P.grid), dim3(kThreads), args, smem, st));
  }
  P.wait = 0;
  const int L = P.num_levels;
  for (int li = 0; li < L; ++li) {
    const int l = bwd ? L - 1 - li : li;
    P.step_begin = T.level_step0[l];
    P.step_end = T.level_step0[l] + T.level_steps[l];
    void* args[] = {&P};
    int err = int(cudaLaunchKernel(fn, dim3(P.grid), dim3(kThreads), args, smem, st));
    if (err) return err;
  }
  return 0;
}

int launch_slack(DevGraph& g, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (g.num_ep == 0) return int(cudaMemsetAsync(g.summary, 0, sizeof(double) * 3, st));
  const int blocks = (g.num_ep + kRedThreads - 1) / kRedThreads;
  slack_kernel<<<blocks, kRedThreads, 0, st>>>(g.num_ep, g.ep_pin, g.ep_rat, g.state,
                                              g.last_n_sigma, g.slack, g.rf_star, g.partials,
                                              g.ticket, g.summary);
  return int(cudaGetLastError());
}

int launch_forward(DevGraph& g, float n_sigma, float tau, int schedule, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  KParams P = make_params(g, false);
  P.n_sigma = n_sigma;
  P.tau = tau;
  const bool lse = tau > 0.f;
  if (g.n > 0) {
    if (schedule == 0) P.epoch = ++g.epoch_fwd;
    int err = launch_items(lse ? (const void*)fwd_kernel<true> : (const void*)fwd_kernel<false>,
                           kFwdSmem, P, g.fwd_items, false, schedule, st);
    if (err) return err;
  }
  g.last_n_sigma = n_sigma;
  g.last_tau = tau;
  return launch_slack(g, stream);
}

int launch_backward(DevGraph& g, const float* ep_seed, float* d_arc_mean, float* d_src,
                    void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaSuccess;
  if (g.e > 0) {
    e = cudaMemsetAsync(d_arc_mean, 0, sizeof(float) * 2 * size_t(g.e), st);
    if (e != cudaSuccess) return int(e);
  }
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
  KParams P = make_params(g, true);
  P.n_sigma = g.last_n_sigma;
  P.tau = g.last_tau;
  P.d_mean = d_arc_mean;
  P.d_src = d_src;
  const bool lse = g.last_tau > 0.f;
  if (g.bwd_schedule == 0) P.epoch = ++g.epoch_bwd;
  return launch_items(lse ? (const void*)bwd_kernel<true> : (const void*)bwd_kernel<false>, kBwdSmem,
                      P, g.bwd_items, true, g.bwd_schedule, st);
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
