// batch.cu -- batched scenario evaluation (BASELINE north
// star: "independent evaluations ... batches of candidate gate-sizing
// perturbations or PVT/OCV scenarios").
//
// Up to kLanes = 32 scenarios are evaluated in one pass over the graph.  The
// per-pin state is scenario-minor ([pin][scenario], 32 B per entry), so the 32
// lanes of a warp are the 32 scenarios of ONE pin: every source-state gather
// is a contiguous 1 KB access, and the topology (row pointers, source words,
// arc records -- TMA-staged per item exactly as in kernels.cu) is read once
// for all scenarios.  Scenario s materializes its arc table in fp32 as the
// oracle does: mean' = fl32(mean * d), sigma' = fl32(sigma *
// d) with d = derate_cell or derate_net by arc class, then sparse overrides
// replace whole arc records; N_sigma is per scenario.  Candidate arithmetic,
// merge order and LSE are the same device functions as the single-scenario
// path, so each scenario's arrivals are bit-identical to insta_forward on the
// materialized graph.  Synchronization is the same parity dataflow.
//
// The optional backward accumulates sum_s dTNS_s / d(arc mean') into one
// [E][2] buffer: per arc, the 32 lanes' contributions are summed by a fixed
// xor-shuffle tree and added by lane 0 (each arc is written by exactly one
// warp per pass, so the read-modify-write needs no atomics).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <cstdint>
#include <vector>

#include "device_common.cuh"
#include "internal.h"

namespace insta {

constexpr int kLanes = 32;
constexpr double kFixB = 16777216.0;          // 2^24 (heavy accumulators, as kernels.cu)
constexpr long long kCountUnitB = 1ll << 44;

struct BParams {
  int32_t n, num_levels, grid, step_begin, step_end, nb;
  int32_t store_aux;   // forward: write the arg-max / Eq 6 weights (only when a backward follows)
  uint32_t par;
  float tau;
  double inv_tau;
  const int4* __restrict__ item_a;
  const int4* __restrict__ item_b;
  const int32_t* __restrict__ fanin_ptr;
  const int32_t* __restrict__ fin_src;
  const float4* __restrict__ fin_ms;
  const uint8_t* __restrict__ fin_flags;   // bit 0: cell arc, bit 1: overridden in this batch
  const int32_t* __restrict__ fin_arc;
  const int32_t* __restrict__ lfo_ptr;
  const int32_t* __restrict__ lfo;
  const int32_t* __restrict__ heavy_slot;
  const int32_t* __restrict__ heavy_fo;
  const int32_t* __restrict__ ep_of_pin;
  const float4* __restrict__ src_ms;
  // stage-folded forward (fold.cpp): head pins and first fanin positions,
  // folded pin word / fanin position / record of e' per entry
  const int32_t* __restrict__ hd_pin;
  const int32_t* __restrict__ hd_q0;
  const int32_t* __restrict__ ext_f;
  const int32_t* __restrict__ ext_fq;
  const float4* __restrict__ ext_fms;
  const int32_t* __restrict__ ext_qpos;      // backward: fanin position of e
  const int32_t* __restrict__ ext_farc;      // backward: caller id of e' (-1: not folded)
  const int32_t* __restrict__ heavy_slot_pin;   // heavy slot per canonical pin (heavy adds)
  const float* __restrict__ sc;            // [3][32]: n_sigma, derate_cell, derate_net
  const int32_t* __restrict__ ov_ptr;      // [33] overrides of scenario s: [ov_ptr[s], ov_ptr[s+1])
  const int32_t* __restrict__ ov_pos;      // arc keys: fanin positions (backward) / entry keys 2x, 2x+1 (forward)
  const float4* __restrict__ ov_ms;        // override arc records
  PinState* bstate;                        // [n][32]
  int32_t* bwin;                           // [n][32]
  float4* bwts;                            // [e][32]
  float2* bg;                              // [e][32]
  unsigned long long* bheavy;              // [heavy][32][2]
  const float* bslack;                     // [P][32]
  const uint8_t* brf;                      // [P][32]
  float* d_mean_sum;                       // [e][2] (accumulated)
};

// ---------------------------------------------------------------- scenario arcs
__device__ __forceinline__ float4 scen_arc(const BParams& P, float4 ms, uint32_t flags, int q, int s,
                                           float dcell, float dnet) {
  if (flags & 2u) {
    for (int o = __ldg(P.ov_ptr + s); o < __ldg(P.ov_ptr + s + 1); ++o)
      if (__ldg(P.ov_pos + o) == q) return __ldg(P.ov_ms + o);
  }
  const float d = (flags & 1u) ? dcell : dnet;
  return make_float4(ms.x * d, ms.y * d, ms.z * d, ms.w * d);
}

__device__ __forceinline__ Raw ldb_raw(const BParams& P, int j, int s) {
  Raw r;
  asm volatile("ld.relaxed.gpu.global.v4.b64 {%0, %1, %2, %3}, [%4];"
               : "=l"(r.a), "=l"(r.b), "=l"(r.c), "=l"(r.d)
               : "l"(P.bstate + size_t(j) * kLanes + s)
               : "memory");
  return r;
}

__device__ __forceinline__ void awaitb(const BParams& P, int j, int s, Raw& r) {
  uint32_t npoll_ = 0;
  while (!raw_ready(r, P.par)) {
    insta_poll_pause(npoll_);
    r = ldb_raw(P, j, s);
  }
}

__device__ __forceinline__ void storeb(const BParams& P, int i, int s, double m0, double m1, double v0,
                                       double v1) {
  asm volatile("st.relaxed.gpu.global.v4.f64 [%0], {%1, %2, %3, %4};" ::"l"(P.bstate + size_t(i) * kLanes + s),
               "d"(with_par(m0, P.par)), "d"(with_par(m1, P.par)), "d"(with_par(v0, P.par)),
               "d"(with_tag(v1, P.par, 0u))
               : "memory");
}

// ---------------------------------------------------------------- forward
// Stage-folded schedule (fold.cpp, as kernels.cu fwd_kernel<., true>): items
// are head ranges per super-level; an entry through a folded pin p first
// computes p for the lane's scenario from the gathered source words (merge1,
// the nf = 1 merge) and stores it, then continues with p's words.  Arc keys
// for the sparse overrides: 2x for the entry's arc e, 2x + 1 for e'.
struct BFwdStage {
  int32_t ptr[kBFwdPins + 8];     // entry rows of the heads
  int32_t pin[kBFwdPins + 8];     // canonical pin of each head
  int32_t src[kBFwdArcs + 8];     // entry source word (fold bit 29)
  int32_t f[kBFwdArcs + 8];       // folded pin | unate(e') << 30
  int32_t fq[kBFwdArcs + 8];      // fanin position of e'
  uint8_t flags[kBFwdArcs + 32];  // bit 0/1: e cell / overridden, bit 2/3: e'
  float4 ms[kBFwdArcs];           // record of e
  float4 fms[kBFwdArcs];          // record of e'
};
constexpr size_t kBFwdSmem = 2 * sizeof(BFwdStage);

__device__ __forceinline__ bool bfwd_staged(const int4& A, const int4& B) {
  return A.y > A.x && B.x > 0 && !(B.y & kItemDirect);
}

__device__ __forceinline__ void bfwd_prefetch(const BParams& P, BFwdStage* st, uint64_t* full, int step, int c) {
  const int4 A = __ldg(P.item_a + size_t(step) * P.grid + c);
  const int4 B = __ldg(P.item_b + size_t(step) * P.grid + c);
  if (!bfwd_staged(A, B)) return;
  const Window wp = window(A.x, A.y + 1, 4);
  const Window wh = window(A.x, A.y, 4);
  const Window ws = window(A.z, A.w, 4);
  const Window wf = window(A.z, A.w, 1);
  const uint32_t bms = uint32_t(A.w - A.z) * 16u;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_expect_tx(full, wp.bytes + wh.bytes + (ws.bytes ? 3 * ws.bytes + wf.bytes + 2 * bms : 0u));
  bulk_g2s(st->ptr, P.fanin_ptr + wp.start, wp.bytes, full);
  bulk_g2s(st->pin, P.hd_pin + wh.start, wh.bytes, full);
  if (ws.bytes) {
    bulk_g2s(st->src, P.fin_src + ws.start, ws.bytes, full);
    bulk_g2s(st->f, P.ext_f + ws.start, ws.bytes, full);
    bulk_g2s(st->fq, P.ext_fq + ws.start, ws.bytes, full);
    bulk_g2s(st->flags, P.fin_flags + wf.start, wf.bytes, full);
    bulk_g2s(st->ms, P.fin_ms + A.z, bms, full);
    bulk_g2s(st->fms, P.ext_fms + A.z, bms, full);
  }
}

// Merge of (pin, rf) for scenario lane s: the same device function as the
// single-scenario kernels (device_common.cuh merge_rf), hence bit-identical.
template <bool kLSE, class ArcFn>
__device__ __forceinline__ RfOut pin_rf_b(const BParams& P, double ns, int rf, int nf, ArcFn&& arc) {
  return merge_rf<kLSE>(ns, double(P.tau), P.inv_tau, rf, nf, arc);
}

template <class ArcFn>
__device__ __forceinline__ float2 arc_rf_weights_b(const BParams& P, double ns, int rf, int k, const RfOut& o,
                                                   ArcFn&& arc) {
  return arc_weights(ns, P.inv_tau, rf, k, o, arc);
}

#ifndef INSTA_BREG
#define INSTA_BREG 3
#endif
constexpr int kRegArcsB = INSTA_BREG;   // source words of a pin's first arcs held in registers

// folded pin p behind entry x for scenario lane s (merge1 = the nf = 1 merge)
// store: also write p's state (entries past the register window, read back by the merge)
template <bool kLSE>
__device__ __forceinline__ Raw foldb(const BParams& P, int32_t fw, int32_t fq, float4 fm, uint32_t fl, int x, int s,
                                  double ns, float dcell, float dnet, Raw rj, bool store) {
  const float4 ms = scen_arc(P, fm, fl >> 2, 2 * x + 1, s, dcell, dnet);
  Merge1 m;
  merge1<kLSE>(unpack(rj), int(uint32_t(fw) >> kUnateShift), ms, ns, double(P.tau), P.inv_tau, m);
  // normally no state store: a folded pin's only consumer is the head
  // computing it here, and batched evaluations report summaries and gradients
  const int pp = fw & kSrcMask;
  if (store) storeb(P, pp, s, m.mu[0], m.mu[1], m.var[0], m.var[1]);
  if (P.store_aux) {
    if (!kLSE) P.bwin[size_t(pp) * kLanes + s] = m.win;
    else P.bwts[size_t(fq) * kLanes + s] = m.wt;
  }
  return m.stored(P.par);
}

template <bool kLSE>
__global__ void __launch_bounds__(kThreads, 1) fwdb_kernel(BParams P) {
  extern __shared__ __align__(128) unsigned char smem[];
  BFwdStage* stage = reinterpret_cast<BFwdStage*>(smem);
  __shared__ __align__(8) uint64_t full[2];
  const int c = blockIdx.x, tid = threadIdx.x;
  const int warp = tid >> 5, s = tid & 31;
  const bool lane_on = s < P.nb;
  const double ns = double(__ldg(P.sc + s));
  const float dcell = __ldg(P.sc + kLanes + s), dnet = __ldg(P.sc + 2 * kLanes + s);
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[0])) : "memory");
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[1])) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  uint32_t phase[2] = {0u, 0u};
  const int nsteps = P.step_end - P.step_begin;
  if (tid == 0 && nsteps > 0) bfwd_prefetch(P, &stage[0], &full[0], P.step_begin, c);
  for (int t = 0; t < nsteps; ++t) {
    const int buf = t & 1, k = P.step_begin + t;
    const int4 A = __ldg(P.item_a + size_t(k) * P.grid + c);
    const int4 B = __ldg(P.item_b + size_t(k) * P.grid + c);
    if (tid == 0 && t + 1 < nsteps) bfwd_prefetch(P, &stage[buf ^ 1], &full[buf ^ 1], k + 1, c);
    if (A.y > A.x) {
      if (B.x == 0) {   // startpoints: heads 0..num_src-1 are canonical pins 0..num_src-1
        for (int i = A.x + warp; i < A.y; i += kThreads / 32) {
          if (!lane_on) continue;
          const float4 v = __ldg(P.src_ms + i);
          storeb(P, i, s, double(v.x), double(v.y), double(v.z) * double(v.z), double(v.w) * double(v.w));
        }
      } else {
        const bool staged = !(B.y & kItemDirect);
        if (staged) {
          mbar_wait(&full[buf], phase[buf]);
          phase[buf] ^= 1u;
        }
        const BFwdStage& S = stage[buf];
        const int po = A.x & 3, so = A.z & 3, fo = A.z & 15;
        for (int p = warp; p < A.y - A.x && lane_on; p += kThreads / 32) {
          const int h = A.x + p;
          int b0, nf, i;
          if (staged) {
            b0 = S.ptr[po + p] - A.z;
            nf = S.ptr[po + p + 1] - A.z - b0;
            i = S.pin[po + p];
          } else {
            b0 = __ldg(P.fanin_ptr + h) - A.z;
            nf = __ldg(P.fanin_ptr + h + 1) - A.z - b0;
            i = __ldg(P.hd_pin + h);
          }
          // entry kk: source word, flags, record of e (and of e' and the folded pin)
          auto ent = [&](int kk, int32_t& w, uint32_t& fl, float4& m0) {
            if (staged) {
              w = S.src[so + b0 + kk];
              fl = S.flags[fo + b0 + kk];
              m0 = S.ms[b0 + kk];
            } else {
              const int x = A.z + b0 + kk;
              w = __ldg(P.fin_src + x);
              fl = __ldg(P.fin_flags + x);
              m0 = __ldg(P.fin_ms + x);
            }
          };
          // folded pin behind entry kk: computed for this scenario from the source words
          auto fold = [&](int kk, uint32_t fl, const Raw& rj, bool store) -> Raw {
            const int x = A.z + b0 + kk;
            if (staged) return foldb<kLSE>(P, S.f[so + b0 + kk], S.fq[so + b0 + kk], S.fms[b0 + kk], fl, x, s, ns,
                                           dcell, dnet, rj, store);
            return foldb<kLSE>(P, __ldg(P.ext_f + x), __ldg(P.ext_fq + x), __ldg(P.ext_fms + x), fl, x, s, ns, dcell,
                               dnet, rj, store);
          };
          // gather the first kRegArcsB source entries of this scenario together
          Raw rr[kRegArcsB];
          auto src_word = [&](int kk) { return staged ? S.src[so + b0 + kk] : __ldg(P.fin_src + A.z + b0 + kk); };
#pragma unroll
          for (int kk = 0; kk < kRegArcsB; ++kk)
            if (kk < nf) rr[kk] = ldb_raw(P, src_word(kk) & kSrcMask, s);
#pragma unroll
          for (int kk = 0; kk < kRegArcsB; ++kk) {
            if (kk < nf) {
              int32_t w;
              uint32_t fl;
              float4 m0;
              ent(kk, w, fl, m0);
              awaitb(P, w & kSrcMask, s, rr[kk]);
              if ((w >> kFoldBit) & 1) rr[kk] = fold(kk, fl, rr[kk], false);
            }
          }
          // entries past the register window: folded pins are computed and stored here once,
          // the merge below reads their words back like any other source
          for (int kk = kRegArcsB; kk < nf; ++kk) {
            int32_t w;
            uint32_t fl;
            float4 m0;
            ent(kk, w, fl, m0);
            if ((w >> kFoldBit) & 1) {
              Raw r = ldb_raw(P, w & kSrcMask, s);
              awaitb(P, w & kSrcMask, s, r);
              fold(kk, fl, r, true);
            }
          }
          auto arc = [&](int kk, int32_t& w, float4& ms, Raw& r) {
            uint32_t fl;
            float4 m0;
            ent(kk, w, fl, m0);
            ms = scen_arc(P, m0, fl & 3u, 2 * (A.z + b0 + kk), s, dcell, dnet);
            if (kk < kRegArcsB) {
              r = rr[0];
#pragma unroll
              for (int x = 1; x < kRegArcsB; ++x)
                if (x == kk) r = rr[x];
            } else {
              // folded: the pin stored above by this lane; else the source
              const int src = ((w >> kFoldBit) & 1) ? ((staged ? S.f[so + b0 + kk] : __ldg(P.ext_f + A.z + b0 + kk)) & kSrcMask)
                                                    : (w & kSrcMask);
              r = ldb_raw(P, src, s);
              awaitb(P, src, s, r);
            }
          };
          RfOut R, F;
          if (nf <= kRegArcsB) {   // register window: unrolled merge, no run-time source selection
            R = merge_rf_unrolled<kLSE, kRegArcsB>(ns, double(P.tau), P.inv_tau, 0, nf, arc);
            F = merge_rf_unrolled<kLSE, kRegArcsB>(ns, double(P.tau), P.inv_tau, 1, nf, arc);
          } else {
            R = pin_rf_b<kLSE>(P, ns, 0, nf, arc);
            F = pin_rf_b<kLSE>(P, ns, 1, nf, arc);
          }
          storeb(P, i, s, R.mu, F.mu, R.var, F.var);
          if (!P.store_aux) {
          } else if (!kLSE) {
            P.bwin[size_t(i) * kLanes + s] = R.win | (F.win << 16);
          } else {
            const int q0 = __ldg(P.hd_q0 + h);
            for (int kk = 0; kk < nf; ++kk) {
              const float2 wr = arc_rf_weights_b(P, ns, 0, kk, R, arc);
              const float2 wf = arc_rf_weights_b(P, ns, 1, kk, F, arc);
              P.bwts[size_t(q0 + kk) * kLanes + s] = make_float4(wr.x, wr.y, wf.x, wf.y);
            }
          }
        }
      }
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- slack
// slack[ep][s] = RAT - A (min over rf, tie -> R); per-scenario WNS/TNS/#viol
// via fixed-order reductions (block partials over endpoints, then the last block).
constexpr int kSlackEps = 8;   // endpoint rows per 256-thread block iteration

__global__ void __launch_bounds__(256) slackb_kernel(int num_ep, int nb, const int32_t* __restrict__ ep_pin,
                                                     const float2* __restrict__ ep_rat,
                                                     const PinState* __restrict__ bstate,
                                                     const float* __restrict__ sc, float* bslack, uint8_t* brf,
                                                     double* partials, uint32_t* ticket, double* summaries) {
  __shared__ double st[3][kSlackEps][kLanes];
  __shared__ bool s_last;
  const int s = threadIdx.x & 31, row = threadIdx.x >> 5;
  const double ns = double(sc[s]);
  double tns = 0.0, wns = 0.0, nv = 0.0;
  const int per_block = kSlackEps * 64;
  const int e0 = blockIdx.x * per_block;
  for (int e = e0 + row; e < min(num_ep, e0 + per_block); e += kSlackEps) {
    if (s >= nb) continue;
    const double2 m = __ldcg(reinterpret_cast<const double2*>(bstate + size_t(ep_pin[e]) * kLanes + s));
    const double2 v = __ldcg(reinterpret_cast<const double2*>(bstate + size_t(ep_pin[e]) * kLanes + s) + 1);
    const float2 rat = ep_rat[e];
    const double aR = strip((unsigned long long)__double_as_longlong(m.x)) +
                      ns * double(sigma_of(strip((unsigned long long)__double_as_longlong(v.x))));
    const double aF = strip((unsigned long long)__double_as_longlong(m.y)) +
                      ns * double(sigma_of(strip2((unsigned long long)__double_as_longlong(v.y))));
    const double sR = double(rat.x) - aR, sF = double(rat.y) - aF;
    const bool fall = sF < sR;
    const double sl = fall ? sF : sR;
    bslack[size_t(e) * kLanes + s] = float(sl);
    brf[size_t(e) * kLanes + s] = fall ? 1 : 0;
    if (sl < 0.0) {
      tns += sl;
      nv += 1.0;
      wns = fmin(wns, sl);
    }
  }
  st[0][row][s] = tns;
  st[1][row][s] = wns;
  st[2][row][s] = nv;
  __syncthreads();
  if (row == 0) {
    for (int r = 1; r < kSlackEps; ++r) {
      tns += st[0][r][s];
      wns = fmin(wns, st[1][r][s]);
      nv += st[2][r][s];
    }
    partials[(size_t(blockIdx.x) * 3 + 0) * kLanes + s] = tns;
    partials[(size_t(blockIdx.x) * 3 + 1) * kLanes + s] = wns;
    partials[(size_t(blockIdx.x) * 3 + 2) * kLanes + s] = nv;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last || row != 0) return;
  __threadfence();
  tns = 0.0;
  wns = 0.0;
  nv = 0.0;
  for (int b = 0; b < int(gridDim.x); ++b) {
    tns += __ldcg(partials + (size_t(b) * 3 + 0) * kLanes + s);
    wns = fmin(wns, __ldcg(partials + (size_t(b) * 3 + 1) * kLanes + s));
    nv += __ldcg(partials + (size_t(b) * 3 + 2) * kLanes + s);
  }
  if (s < nb) {
    summaries[size_t(s) * 3 + 0] = wns;
    summaries[size_t(s) * 3 + 1] = tns;
    summaries[size_t(s) * 3 + 2] = nv;
  }
  if (s == 0) *ticket = 0u;
}

// ---------------------------------------------------------------- backward
// Stage-folded schedule (as kernels.cu bwdf_kernel): items are head ranges in
// reverse super-level order, one warp per head, one lane per scenario.  The
// head's adjoint is pulled from its light fanout rows (all loads of a chunk
// issued before any is checked) + heavy accumulator + TNS seed; each entry
// applies the Eq 6 sink side of its arc e and, through a folded pin p, of e'
// (p's adjoint = what its own pull would form: 0 + ((0 + g) + 0), g with the
// parity LSB cleared).  Bit-identical per scenario to the per-level schedule.
struct BBwdStage {
  int32_t lptr[kBwdPins + 8];   // light fanout rows of the heads
  int32_t lfo[kBwdFanout + 8];  // adjoint word positions of those rows
  int32_t fptr[kBwdPins + 8];   // entry rows of the heads
  int32_t pin[kBwdPins + 8];    // canonical pin of each head
  int32_t hslot[kBwdPins + 8];  // heavy accumulator slot (-1: light)
  int32_t eop[kBwdPins + 8];    // endpoint index of the head (-1: none)
  int32_t qpos[kBwdArcs + 8];   // fanin position of e
  int32_t src[kBwdArcs + 8];    // fin_src word of the arc whose adjoint the entry writes
  int32_t arc[kBwdArcs + 8];    // caller id of e
  int32_t farc[kBwdArcs + 8];   // caller id of e' (-1: not folded)
  int32_t fq[kBwdArcs + 8];     // fanin position of e'
  int32_t f[kBwdArcs + 8];      // folded pin word
};
constexpr size_t kBBwdSmem = 2 * sizeof(BBwdStage);

__device__ __forceinline__ void bbwd_prefetch(const BParams& P, BBwdStage* st, uint64_t* full, int step, int c) {
  const int4 A = __ldg(P.item_a + size_t(step) * P.grid + c);   // {h_lo, h_hi, lfo_lo, lfo_hi}
  const int4 B = __ldg(P.item_b + size_t(step) * P.grid + c);   // {x_lo, x_hi, slevel, flags}
  if (!(A.y > A.x && !(B.w & kItemDirect))) return;
  const Window wl = window(A.x, A.y + 1, 4);
  const Window wf = window(A.z, A.w, 4);
  const Window wa = window(B.x, B.y, 4);
  const Window wh = window(A.x, A.y, 4);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_expect_tx(full, 2 * wl.bytes + wf.bytes + 6 * wa.bytes + 3 * wh.bytes);
  bulk_g2s(st->lptr, P.lfo_ptr + wl.start, wl.bytes, full);
  if (wf.bytes) bulk_g2s(st->lfo, P.lfo + wf.start, wf.bytes, full);
  bulk_g2s(st->fptr, P.fanin_ptr + wl.start, wl.bytes, full);
  bulk_g2s(st->pin, P.hd_pin + wh.start, wh.bytes, full);
  bulk_g2s(st->hslot, P.heavy_slot + wh.start, wh.bytes, full);
  bulk_g2s(st->eop, P.ep_of_pin + wh.start, wh.bytes, full);
  if (wa.bytes) {
    bulk_g2s(st->qpos, P.ext_qpos + wa.start, wa.bytes, full);
    bulk_g2s(st->src, P.fin_src + wa.start, wa.bytes, full);
    bulk_g2s(st->arc, P.fin_arc + wa.start, wa.bytes, full);
    bulk_g2s(st->farc, P.ext_farc + wa.start, wa.bytes, full);
    bulk_g2s(st->fq, P.ext_fq + wa.start, wa.bytes, full);
    bulk_g2s(st->f, P.ext_f + wa.start, wa.bytes, full);
  }
}

__device__ __forceinline__ bool g_ready(uint32_t a, uint32_t b, uint32_t par) {
  return ((a & 1u) == par) && ((b & 1u) == par);
}

__device__ __forceinline__ float2 loadb_g(const BParams& P, int q, int s) {
  uint32_t a, b;
  const float2* p = P.bg + size_t(q) * kLanes + s;
  ld2_u32(p, a, b);
  uint32_t npoll_ = 0;
  while (!g_ready(a, b, P.par)) {
    insta_poll_pause(npoll_);
    ld2_u32(p, a, b);
  }
  return make_float2(stripf(a), stripf(b));
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int d = 16; d >= 1; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
  return v;
}

// Eq 6 sink side of one arc for this lane's scenario: weights from the
// arg-max word (hard, fanin index kk) or the stored weights (LSE) at fanin
// position q.  Returns the adjoint to the source; writes the scenario-summed
// dL/d(arc mean) (lane 0, one warp per arc per pass: plain read-modify-write).
template <bool kLSE>
__device__ __forceinline__ float2 bsink(const BParams& P, bool lane_on, int s, float2 ab, int32_t win, int kk, int q,
                                        int32_t arcid) {
  float w[2][2] = {{0.f, 0.f}, {0.f, 0.f}};
  if (lane_on) {
    if (kLSE) {
      const float4 w4 = P.bwts[size_t(q) * kLanes + s];
      w[0][0] = w4.x;
      w[0][1] = w4.y;
      w[1][0] = w4.z;
      w[1][1] = w4.w;
    } else {
#pragma unroll
      for (int rf = 0; rf < 2; ++rf) {
        const int wv = (win >> (16 * rf)) & 0xffff;
        const bool hit = (wv & 0x7fff) == kk;
        w[rf][0] = (hit && (wv >> 15) == 0) ? 1.f : 0.f;
        w[rf][1] = (hit && (wv >> 15) == 1) ? 1.f : 0.f;
      }
    }
  }
  const float abr[2] = {ab.x, ab.y};
  float gm[2], gs[2] = {0.f, 0.f};
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    const float a0 = w[rf][0] * abr[rf], a1 = w[rf][1] * abr[rf];
    gm[rf] = a0 + a1;
    gs[0] += a0;
    gs[1] += a1;
  }
  // sum over scenarios of dTNS_s/d(arc mean'), fixed xor tree
  const float t0 = warp_sum(gm[0]), t1 = warp_sum(gm[1]);
  if (s == 0 && (t0 != 0.f || t1 != 0.f)) {
    float2* o = reinterpret_cast<float2*>(P.d_mean_sum) + arcid;
    const float2 prev = *o;
    *o = make_float2(prev.x + t0, prev.y + t1);
  }
  return make_float2(gs[0], gs[1]);
}

// publish the adjoint of the arc at fanin position q to its source (srcw)
__device__ __forceinline__ void bpublish(const BParams& P, int s, int q, int32_t srcw, float2 gs) {
  st2_f32(P.bg + size_t(q) * kLanes + s, with_parf(gs.x, P.par), with_parf(gs.y, P.par));
  if ((srcw >> kHeavyBit) & 1) {
    const int hs = __ldg(P.heavy_slot_pin + (srcw & kSrcMask));
    unsigned long long* acc = P.bheavy + (size_t(hs) * kLanes + s) * 2;
    atomicAdd(acc, (unsigned long long)(kCountUnitB + __double2ll_rn(double(gs.x) * kFixB)));
    atomicAdd(acc + 1, (unsigned long long)(kCountUnitB + __double2ll_rn(double(gs.y) * kFixB)));
  }
}

constexpr int kPullChunk = 4;

template <bool kLSE>
__global__ void __launch_bounds__(kThreads, 1) bwdb_kernel(BParams P) {
  extern __shared__ __align__(128) unsigned char smem[];
  BBwdStage* stage = reinterpret_cast<BBwdStage*>(smem);
  __shared__ __align__(8) uint64_t full[2];
  const int c = blockIdx.x, tid = threadIdx.x;
  const int warp = tid >> 5, s = tid & 31;
  const bool lane_on = s < P.nb;
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[0])) : "memory");
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[1])) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  uint32_t phase[2] = {0u, 0u};
  const int nsteps = P.step_end - P.step_begin;
  if (tid == 0 && nsteps > 0) bbwd_prefetch(P, &stage[0], &full[0], P.step_begin, c);
  for (int t = 0; t < nsteps; ++t) {
    const int buf = t & 1, k = P.step_begin + t;
    const int4 A = __ldg(P.item_a + size_t(k) * P.grid + c);
    const int4 B = __ldg(P.item_b + size_t(k) * P.grid + c);
    const int l = B.z;
    if (tid == 0 && t + 1 < nsteps) bbwd_prefetch(P, &stage[buf ^ 1], &full[buf ^ 1], k + 1, c);
    if (A.y > A.x) {
      const bool staged = !(B.w & kItemDirect);
      if (staged) {
        mbar_wait(&full[buf], phase[buf]);
        phase[buf] ^= 1u;
      }
      const BBwdStage& S = stage[buf];
      const int lo = A.x & 3, fo = A.z & 3, ao = B.x & 3;
      for (int p = warp; p < A.y - A.x; p += kThreads / 32) {
        const int h = A.x + p;
        const int r0 = (staged ? S.lptr[lo + p] : __ldg(P.lfo_ptr + h)) - (staged ? A.z : 0);
        const int r1 = (staged ? S.lptr[lo + p + 1] : __ldg(P.lfo_ptr + h + 1)) - (staged ? A.z : 0);
        const int slot = staged ? S.hslot[lo + p] : __ldg(P.heavy_slot + h);
        const int ep = staged ? S.eop[lo + p] : __ldg(P.ep_of_pin + h);
        const int i = staged ? S.pin[lo + p] : __ldg(P.hd_pin + h);
        float ax = 0.f, ay = 0.f;
        if (lane_on) {
          // pull (row order, fixed): each chunk's loads issued before any is checked
          for (int r = r0; r < r1; r += kPullChunk) {
            uint32_t va[kPullChunk], vb[kPullChunk];
            int qq[kPullChunk];
#pragma unroll
            for (int j = 0; j < kPullChunk; ++j) {
              if (r + j < r1) {
                qq[j] = staged ? S.lfo[fo + r + j] : __ldg(P.lfo + r + j);
                ld2_u32(P.bg + size_t(qq[j]) * kLanes + s, va[j], vb[j]);
              }
            }
#pragma unroll
            for (int j = 0; j < kPullChunk; ++j) {
              if (r + j < r1) {
                uint32_t npoll_ = 0;
                while (!g_ready(va[j], vb[j], P.par)) {
                  insta_poll_pause(npoll_);
                  ld2_u32(P.bg + size_t(qq[j]) * kLanes + s, va[j], vb[j]);
                }
                ax += stripf(va[j]);
                ay += stripf(vb[j]);
              }
            }
          }
          if (slot >= 0) {
            unsigned long long* acc = P.bheavy + (size_t(slot) * kLanes + s) * 2;
            const long long target = __ldg(P.heavy_fo + slot);
            unsigned long long x, y;
            ld2_u64(acc, x, y);
            uint32_t npoll_ = 0;
            while (((long long)x + (kCountUnitB >> 1)) >> 44 != target ||
                   ((long long)y + (kCountUnitB >> 1)) >> 44 != target) {
              insta_poll_pause(npoll_);
              ld2_u64(acc, x, y);
            }
            asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %1};" ::"l"(acc), "l"(0ull) : "memory");
            ax += float(double((long long)x - target * kCountUnitB) / kFixB);
            ay += float(double((long long)y - target * kCountUnitB) / kFixB);
          }
          float sx = 0.f, sy = 0.f;
          if (ep >= 0) {   // TNS seed: dL/dA[rf*] = -1 where slack < 0
            const float sl = P.bslack[size_t(ep) * kLanes + s];
            if (sl < 0.f) {
              if (P.brf[size_t(ep) * kLanes + s]) sy = -1.f;
              else sx = -1.f;
            }
          }
          ax = sx + ax;
          ay = sy + ay;
        }
        if (l == 0) continue;
        const int b0 = staged ? S.fptr[lo + p] - B.x : __ldg(P.fanin_ptr + h) - B.x;
        const int nf = (staged ? S.fptr[lo + p + 1] : __ldg(P.fanin_ptr + h + 1)) - B.x - b0;
        const int32_t win = (!kLSE && lane_on) ? P.bwin[size_t(i) * kLanes + s] : 0;
        for (int kk = 0; kk < nf; ++kk) {   // warp-uniform loop (same head in all lanes)
          const int xr = b0 + kk, x = B.x + xr;
          const int q = staged ? S.qpos[ao + xr] : __ldg(P.ext_qpos + x);
          const int32_t srcw = staged ? S.src[ao + xr] : __ldg(P.fin_src + x);
          const int32_t arcid = staged ? S.arc[ao + xr] : __ldg(P.fin_arc + x);
          const int32_t farc = staged ? S.farc[ao + xr] : __ldg(P.ext_farc + x);
          const float2 gs = bsink<kLSE>(P, lane_on, s, make_float2(ax, ay), win, kk, q, arcid);
          if (farc < 0) {
            if (lane_on) bpublish(P, s, q, srcw, gs);
          } else {   // folded pin: its adjoint as its own pull would form it, then arc e'
            const int fq = staged ? S.fq[ao + xr] : __ldg(P.ext_fq + x);
            const int pp = (staged ? S.f[ao + xr] : __ldg(P.ext_f + x)) & kSrcMask;
            float px = 0.f, py = 0.f;
            px += stripf(__float_as_uint(with_parf(gs.x, P.par)));
            py += stripf(__float_as_uint(with_parf(gs.y, P.par)));
            const float2 abp = make_float2(0.f + (px + 0.f), 0.f + (py + 0.f));
            const int32_t pwin = (!kLSE && lane_on) ? P.bwin[size_t(pp) * kLanes + s] : 0;
            const float2 g2 = bsink<kLSE>(P, lane_on, s, abp, pwin, 0, fq, farc);
            if (lane_on) bpublish(P, s, fq, srcw, g2);
          }
        }
      }
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- flags scatter
__global__ void set_flag_kernel(int n, const int32_t* __restrict__ pos, uint8_t* flags, uint8_t bit, int on) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  if (on) flags[pos[k]] |= bit;
  else flags[pos[k]] &= uint8_t(~bit);
}

// entry-space keys 2x (arc e) / 2x + 1 (arc e'): overridden bit 1 / bit 3
// Override bits of entry x: bit 1 (arc e of the entry) or bit 3 (arc e' of
// its folded pin).  Two keys of one micro-batch can hit the same byte (a cell
// arc and the input net arc behind its folded pin), so the byte is updated
// with a 32-bit atomic on its aligned word (a plain read-modify-write of the
// byte could lose the other key's bit).
__global__ void set_xflag_kernel(int n, const int32_t* __restrict__ key, uint8_t* flags, int on) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  const int x = key[k] >> 1;
  const uint32_t bit = (key[k] & 1) ? 8u : 2u;
  const uintptr_t addr = reinterpret_cast<uintptr_t>(flags + x);
  unsigned int* word = reinterpret_cast<unsigned int*>(addr & ~uintptr_t(3));
  const uint32_t sh = uint32_t(addr & 3) * 8u;
  if (on) atomicOr(word, bit << sh);
  else atomicAnd(word, ~(bit << sh));
}

// ---------------------------------------------------------------- host side
template <class K>
static int set_smem_b(K kernel, size_t bytes) {
  return int(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bytes)));
}

static int ensure_batch(DevGraph& g, bool lse, bool grad) {
  static bool attrs = false;
  if (!attrs) {
    int err = set_smem_b(fwdb_kernel<false>, kBFwdSmem);
    if (!err) err = set_smem_b(fwdb_kernel<true>, kBFwdSmem);
    if (!err) err = set_smem_b(bwdb_kernel<false>, kBBwdSmem);
    if (!err) err = set_smem_b(bwdb_kernel<true>, kBBwdSmem);
    if (err) return err;
    attrs = true;
  }
  // cudaMemset runs on the legacy default stream, which the caller's (torch,
  // non-blocking) stream does not wait for: synchronize once after any
  // allocation so the first pass never sees the buffers before they are zeroed
  // (the parity dataflow would otherwise wait on words the memset overwrites).
  bool fresh = false;
  auto alloc = [&fresh](void** p, size_t bytes) -> int {
    if (*p) return 0;
    cudaError_t e = cudaMalloc(p, bytes + 64);
    if (e != cudaSuccess) return int(e);
    fresh = true;
    return int(cudaMemset(*p, 0, bytes + 64));
  };
  const size_t n = size_t(std::max(g.n, 1)), e = size_t(std::max<int64_t>(g.e, 1));
  int err = alloc(reinterpret_cast<void**>(&g.b_state), n * kLanes * sizeof(PinState));
  if (!err) err = alloc(reinterpret_cast<void**>(&g.b_slack), size_t(std::max(g.num_ep, 1)) * kLanes * sizeof(float));
  if (!err) err = alloc(reinterpret_cast<void**>(&g.b_rf), size_t(std::max(g.num_ep, 1)) * kLanes);
  if (!err) err = alloc(reinterpret_cast<void**>(&g.b_partials),
                        size_t((g.num_ep + kSlackEps * 64 - 1) / (kSlackEps * 64) + 1) * 3 * kLanes * sizeof(double));
  if (!err) err = alloc(reinterpret_cast<void**>(&g.b_ticket), sizeof(uint32_t));
  if (!err && !lse) err = alloc(reinterpret_cast<void**>(&g.b_win), n * kLanes * sizeof(int32_t));
  if (!err && lse) err = alloc(reinterpret_cast<void**>(&g.b_wts), e * kLanes * sizeof(float4));
  if (!err && grad) err = alloc(reinterpret_cast<void**>(&g.b_g), e * kLanes * sizeof(float2));
  if (!err && grad) err = alloc(reinterpret_cast<void**>(&g.b_heavy),
                                size_t(std::max(g.num_heavy, 1)) * kLanes * 2 * sizeof(unsigned long long));
  if (!err && fresh) err = int(cudaDeviceSynchronize());
  return err;
}

static BParams make_bparams(DevGraph& g, bool bwd) {
  BParams P{};
  P.n = g.n;
  P.num_levels = g.num_levels;
  P.grid = g.grid;
  P.item_a = bwd ? g.bwdf_a : g.bfwdf_a;
  P.item_b = bwd ? g.bwdf_b : g.bfwdf_b;
  P.fanin_ptr = g.hd_ptr;
  P.fin_src = bwd ? g.ext_bw : g.ext_w;
  P.fin_ms = g.ext_ms;
  P.fin_flags = bwd ? g.fin_flags : g.ext_flags;
  P.ext_qpos = g.ext_qpos;
  P.ext_farc = g.ext_farc;
  P.hd_pin = g.hd_pin;
  P.hd_q0 = g.hd_q0;
  P.ext_f = g.ext_f;
  P.ext_fq = g.ext_fq;
  P.ext_fms = g.ext_fms;
  P.fin_arc = bwd ? g.ext_arc : g.fin_arc;
  P.lfo_ptr = g.hlfo_ptr;
  P.lfo = g.hlfo;
  P.heavy_slot = bwd ? g.hd_hslot : g.heavy_slot;   // backward: per head (staged); heavy_add uses hslot_pin
  P.heavy_slot_pin = g.heavy_slot;
  P.heavy_fo = g.heavy_fo;
  P.ep_of_pin = bwd ? g.hd_eop : g.ep_of_pin;
  P.src_ms = g.src_ms;
  P.bstate = g.b_state;
  P.bwin = g.b_win;
  P.bwts = g.b_wts;
  P.bg = g.b_g;
  P.bheavy = g.b_heavy;
  P.bslack = g.b_slack;
  P.brf = g.b_rf;
  return P;
}

int batch_stage(DevGraph& g, const void* host, size_t bytes, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaSuccess;
  if (!g.b_stage_copied) e = cudaEventCreateWithFlags(reinterpret_cast<cudaEvent_t*>(&g.b_stage_copied), cudaEventDisableTiming);
  if (e == cudaSuccess && !g.b_stage_done)
    e = cudaEventCreateWithFlags(reinterpret_cast<cudaEvent_t*>(&g.b_stage_done), cudaEventDisableTiming);
  if (e != cudaSuccess) return int(e);
  // the previous call's kernels may still read the device copy (possibly on another stream), and
  // its H2D copy may still read the pinned buffer
  e = cudaStreamWaitEvent(st, static_cast<cudaEvent_t>(g.b_stage_done), 0);
  if (e == cudaSuccess) e = cudaEventSynchronize(static_cast<cudaEvent_t>(g.b_stage_copied));
  if (e == cudaSuccess && bytes > g.b_stage_cap) {
    e = cudaStreamSynchronize(st);
    if (e == cudaSuccess && g.b_stage) e = cudaFree(g.b_stage);
    if (e == cudaSuccess && g.b_stage_h) e = cudaFreeHost(g.b_stage_h);
    g.b_stage = nullptr;
    g.b_stage_h = nullptr;
    g.b_stage_cap = 0;
    const size_t cap = std::max<size_t>(bytes + bytes / 2, 1 << 16);
    if (e == cudaSuccess) e = cudaMalloc(&g.b_stage, cap);
    if (e == cudaSuccess) e = cudaMallocHost(&g.b_stage_h, cap);
    if (e == cudaSuccess) g.b_stage_cap = cap;
  }
  if (e != cudaSuccess) return int(e);
  std::memcpy(g.b_stage_h, host, bytes);
  e = cudaMemcpyAsync(g.b_stage, g.b_stage_h, bytes, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaEventRecord(static_cast<cudaEvent_t>(g.b_stage_copied), st);
  return int(e);
}

int batch_stage_release(DevGraph& g, void* stream) {
  return int(cudaEventRecord(static_cast<cudaEvent_t>(g.b_stage_done), static_cast<cudaStream_t>(stream)));
}

int launch_forward_batch(DevGraph& g, const BatchSlice& bs, float tau, double* summaries, float* d_mean_sum,
                         void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const bool lse = tau > 0.f, grad = d_mean_sum != nullptr;
  const int nb = bs.nb, nov = bs.nov;
  int err = ensure_batch(g, lse, grad);
  if (err) return err;
  cudaError_t e = cudaSuccess;
  if (nov > 0) {
    set_flag_kernel<<<(nov + 255) / 256, 256, 0, st>>>(nov, bs.ov_pos, g.fin_flags, 2, 1);
    set_xflag_kernel<<<(nov + 255) / 256, 256, 0, st>>>(nov, bs.ov_key, g.ext_flags, 1);
    e = cudaGetLastError();
  }
  if (e != cudaSuccess) return int(e);
  BParams P = make_bparams(g, false);
  P.sc = bs.sc;
  P.ov_ptr = bs.ov_ptr;
  P.ov_pos = bs.ov_key;
  P.ov_ms = bs.ov_ms;
  P.nb = nb;
  P.tau = tau;
  P.inv_tau = lse ? 1.0 / double(tau) : 0.0;
  P.par = (++g.pass_bfwd) & 1u;
  P.store_aux = grad ? 1 : 0;
  P.step_begin = 0;
  P.step_end = g.bfwdf_items.num_steps;
  if (g.n > 0) {
    void* args[] = {&P};
    e = cudaLaunchCooperativeKernel(lse ? (const void*)fwdb_kernel<true> : (const void*)fwdb_kernel<false>,
                                    dim3(g.grid), dim3(kThreads), args, kBFwdSmem, st);
    if (e != cudaSuccess) return int(e);
  }
  if (g.num_ep > 0) {
    const int blocks = (g.num_ep + kSlackEps * 64 - 1) / (kSlackEps * 64);
    slackb_kernel<<<blocks, 256, 0, st>>>(g.num_ep, nb, g.ep_pin, g.ep_rat, g.b_state, bs.sc, g.b_slack, g.b_rf,
                                          g.b_partials, g.b_ticket, summaries);
    e = cudaGetLastError();
  } else {
    e = cudaMemsetAsync(summaries, 0, sizeof(double) * 3 * nb, st);
  }
  if (e != cudaSuccess) return int(e);
  if (grad && g.n > 0) {
    BParams Q = make_bparams(g, true);
    Q.sc = bs.sc;
    Q.ov_ptr = bs.ov_ptr;
    Q.ov_pos = bs.ov_pos;
    Q.ov_ms = bs.ov_ms;
    Q.nb = nb;
    Q.tau = tau;
    Q.inv_tau = P.inv_tau;
    Q.par = (++g.pass_bbwd) & 1u;
    Q.d_mean_sum = d_mean_sum;
    Q.step_begin = 0;
    Q.step_end = g.bwdf_items.num_steps;
    void* args[] = {&Q};
    e = cudaLaunchCooperativeKernel(lse ? (const void*)bwdb_kernel<true> : (const void*)bwdb_kernel<false>,
                                    dim3(g.grid), dim3(kThreads), args, kBBwdSmem, st);
    if (e != cudaSuccess) return int(e);
  }
  if (nov > 0) {
    set_flag_kernel<<<(nov + 255) / 256, 256, 0, st>>>(nov, bs.ov_pos, g.fin_flags, 2, 0);
    set_xflag_kernel<<<(nov + 255) / 256, 256, 0, st>>>(nov, bs.ov_key, g.ext_flags, 0);
    e = cudaGetLastError();
  }
  return int(e);
}

}  // namespace insta
