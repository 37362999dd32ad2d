// sweep.cu -- the persistent passes of the INSTA hot path on the stage-folded
// schedule (schedule 0, the default).
//
// The stage-folded schedule (fold.cpp) groups the pins into "heads" by
// super-level; a netlist's cell input pins are folded into the work of the
// cell output that consumes them, so one (net arc, cell arc) stage costs one
// dependent step (C4: 162 timing levels -> 82 super-levels, every head has at
// most 4 entries).  ONE persistent cooperative launch runs a whole pass: CTA c
// owns the c-th contiguous slice of every super-level's heads and entries.  The
// paper launches one kernel per timing level with a thread per output pin
// (P:L113, L123); this replaces the launch chain by one persistent launch and
// halves the chain length by folding.
//
// Topology staging: a CTA's slice of a level is contiguous in every head- and
// entry-ordered array, so one thread stages the slice of the next level with
// TMA bulk copies (cp.async.bulk + mbarrier) while the current one runs.
//
//  * forward, full pass (fwdx_kernel): per super-level an entry phase (a thread
//    per entry: gather, folded pin, both transitions' Eq 1-3 candidates into
//    shared-memory slots) and a head phase (a thread per head: the first
//    arg-max of Alg 1 / Alg 2, strict ">", or the LSE smooth max
//    of Eq 4; the store); kFlow: no grid barrier, gathers re-poll
//    until the record carries this pass's parity (dataflow), the next level's
//    arc records prefetched to L2.  Folded pins are evaluated in registers and
//    not stored: insta_arrivals and the sigma channel materialize them on
//    demand (fold_fill_kernel).
//  * cone pass (fwdl_kernel, modes 1 / 2): visits only
//    super-levels flagged by a stamped or changed source, recomputes the dirty
//    heads (thread per head), compares each new record with the previous one
//    bitwise and marks the consumers of a changed one; a level with no flag is
//    skipped without a barrier.
//  * candidate evaluation (eval_kernel; C5 sizing candidates): apply, cone
//    pass, the flagged slack blocks, undo log, per candidate in one launch.
//  * backward (bwdl_kernel): Eq 6 weights chained in reverse super-level order
//    (P:L138, L152), push form with int64 fixed-point accumulators (2^-32 ps;
//    exact, order-independent, deterministic), a grid barrier per level.
//  * incremental backward (bdiff_kernel + bwdi_kernel; NEXT 3): fixed-point
//    share deltas over the reverse cone of what changed since a snapshot --
//    bit-identical to the full backward.
//
// Every 64-bit state word carries the pass parity in its LSB (stored values
// are truncated by <= 1 ulp identically in every schedule), so all schedules
// produce the same arrivals bit for bit.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstddef>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>

#include "device_common.cuh"
#include "internal.h"
#include "slack_common.cuh"

namespace insta {

#ifndef INSTA_SL_FWD_THREADS
#define INSTA_SL_FWD_THREADS 384
#endif
#ifndef INSTA_SL_BWD_THREADS
#define INSTA_SL_BWD_THREADS 768
#endif
constexpr int kSLFwdThreads = INSTA_SL_FWD_THREADS;   // forward: ~128-168 registers per thread, 1 CTA / SM
constexpr int kSLBwdThreads = INSTA_SL_BWD_THREADS;   // backward: 1 CTA / SM (768 measured best of 512 / 768 / 1024)
constexpr int kSLNf = 4;                              // entries per head held in registers (netlists: <= 4)
constexpr double kAccScale = 4294967296.0;            // 2^32: fixed-point unit of the backward accumulators
constexpr double kAccInv = 1.0 / 4294967296.0;

struct SLParams {
  int32_t num_sl, num_src, num_heads;
  const int32_t* __restrict__ sl_ptr;
  const int4* __restrict__ slice;        // [SL][grid] {a, b, xa, xb}: CTA c's heads [a, b) of a level, entries [xa, xb)
  const int32_t* __restrict__ hd_ptr;
  const int32_t* __restrict__ hd_pin;
  const int32_t* __restrict__ hd_q0;
  const int32_t* __restrict__ ext_w;
  const float4* ext_ms;                  // written by insta_update_arcs between passes
  const int32_t* __restrict__ ext_f;
  const float4* ext_fms;
  const int32_t* __restrict__ ext_fq;
  const float4* __restrict__ src_ms;
  PinState* state;
  int32_t* win;                          // [n] canonical arg-max words (folded pins, fold_fill)
  float4* wts;                           // [e] canonical Eq 6 weights (folded pins, fold_fill)
  int32_t* hwin;                         // [H] arg-max word of each head (hard mode)
  float4* ew;                            // [X] Eq 6 weights of each entry's arc e (LSE)
  int32_t* fwin;                         // [X] arg-max word of a non-unate folded pin (hard)
  float4* efw;                           // [X] Eq 6 weights of a non-unate folded pin's arc e' (LSE)
  uint32_t* bar;                         // [0] barrier arrivals, [1] exits
  float n_sigma, tau;
  double inv_tau;
  uint32_t par;                          // parity stored in the words' LSB (compatibility with schedule 2)
  int32_t store_fold;                    // 1: also store folded pins' records (fold_fill)
  // cone pass
  uint32_t* dirty;                       // [H] == stamp: recompute
  uint32_t stamp;
  const int32_t* __restrict__ hd_csl;     // [H] consumer super-level range (min | max << 16, -1 none)
  const int32_t* __restrict__ hfo_ptr;    // [H+1] consumer heads (deduplicated rows)
  const int32_t* __restrict__ hfo;
  const int32_t* __restrict__ hfo_sl;     // super-level of each hfo entry
  const uint8_t* __restrict__ hd_hsrc;    // [H] a source of the head has a long consumer row
  uint32_t* chg;                          // [n] == stamp: the pin's record changed in this cone pass
  uint32_t* sl_cnt;                      // [SL] level marked (cleared by the pass)
  unsigned long long* counters;          // [0] pins recomputed
  // backward
  const int32_t* __restrict__ ext_arc;
  const int32_t* __restrict__ ext_farc;
  const int32_t* __restrict__ ext_sh;
  const int32_t* __restrict__ ext_bw;
  const int32_t* __restrict__ order;
  const float2* hseed;
  long long* acc;                        // [H][2]
  float* d_mean;
  float* d_src;
  unsigned long long* trace;             // debug (INSTA_SL_TRACE)
  // endpoint slack (cone passes: the slack blocks holding a changed endpoint are flagged)
  const int32_t* __restrict__ hd_eop;    // [H] endpoint index of the head, -1 none
  uint32_t* ep_blk;                      // [ceil(slack_nb / 32)] flagged slack blocks, or nullptr
  int32_t slack_nb, num_ep;
  const int32_t* __restrict__ ep_pin;
  const float2* __restrict__ ep_rat;
  float* slack;
  uint8_t* rf_star;
  double* partials;
  // candidate evaluation (eval_kernel): arc record arrays and the candidates
  const int32_t* __restrict__ arc_pos;
  const int32_t* __restrict__ arc_xpos;
  const int32_t* __restrict__ arc_head;
  float4* fin_ms;
  float4* ext_ms_w;
  float4* ext_fms_w;
  const int32_t* __restrict__ cand_ptr;  // [n + 1] (device copy)
  const int32_t* __restrict__ cand_arc;
  const float2* __restrict__ cand_m;
  const float2* __restrict__ cand_s;
  float4* cand_old;                      // [arcs of all candidates] saved records
  double* cand_out;                      // [n][3]
  int32_t num_cand;
  // entry-parallel forward (fwdx_kernel): per-CTA candidate buffers in global memory
  // for slices with more than kXCap entries ([grid][xscr_cap] XCand pairs, then bytes)
  void* xscr;
  int32_t xscr_cap;
  // incremental backward (bwdi_kernel) and the snapshot written by a full backward
  long long* acc_b;
  float2* hab_b;
  float2* hseed_b;
  int32_t* hwin_b;
  int32_t* fwin_b;
  float4* ew_b;
  float4* efw_b;
  uint32_t* btouch;   // cone passes stamp the heads they recompute (== bepoch)
  uint32_t bepoch;
  uint32_t* bdirty;
  uint32_t* bl_cnt;
  uint32_t bstamp;
  // eval_kernel undo log (hard mode): a cone pass records what it overwrites
  struct EvLog* elog;        // [elog_cap] head entries
  int2* flog;                // [elog_cap] {entry, old arg-max word} of non-unate folded pins
  uint32_t* elog_n;          // [2] entry counts of this candidate
  int32_t elog_cap;
};

// one undo record: a recomputed head's previous record and arg-max word
struct EvLog {
  Raw rec;
  int32_t pin, h, win, pad;
};

// --------------------------------------------------------------------------
// Grid barrier of the persistent launch: CTA barrier, one release arrival per
// CTA, acquire poll by one thread, CTA barrier.  The counter starts at 0 in
// every launch: the last CTA to leave resets it (grid_exit).
// --------------------------------------------------------------------------
__device__ __forceinline__ void grid_sync_ctr(uint32_t* bar, uint32_t target, unsigned long long* trace) {
  __syncthreads();
  if (threadIdx.x == 0) {
    // trace layout: [0, 512) CTA 0's barrier exits; [512 + k * grid + cta] arrival of cta at barrier k
    if (trace) trace[512 + size_t(target / gridDim.x) * gridDim.x + blockIdx.x] = gtimer();
#ifndef INSTA_SL_NOBAR
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(bar) : "memory");
    uint32_t v, npoll = 0;
    for (;;) {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
      if (v >= target) break;
      if (++npoll > (1u << 23)) __trap();   // bounded: never a silent hang
    }
#endif
    if (trace && blockIdx.x == 0) trace[target / gridDim.x] = gtimer();
  }
  __syncthreads();
}

// barrier number k (1, 2, ...) of this launch
__device__ __forceinline__ void grid_sync(uint32_t* bar, uint32_t k, unsigned long long* trace) {
  grid_sync_ctr(bar, k * gridDim.x, trace);
}

__device__ __forceinline__ void grid_exit(uint32_t* bar) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t prev = atomicAdd(bar + 1, 1u);
    if (prev == gridDim.x - 1) {   // every CTA is past its last barrier poll
      bar[0] = 0u;
      bar[1] = 0u;
    }
  }
}

__device__ __forceinline__ Raw ld_raw(const PinState* p) {
  Raw r;
  asm volatile("ld.relaxed.gpu.global.v4.b64 {%0, %1, %2, %3}, [%4];"
               : "=l"(r.a), "=l"(r.b), "=l"(r.c), "=l"(r.d)
               : "l"(p));
  return r;
}

__device__ __forceinline__ void st_state(PinState* p, double m0, double m1, double v0, double v1, uint32_t par) {
  asm volatile("st.relaxed.gpu.global.v4.f64 [%0], {%1, %2, %3, %4};" ::"l"(p), "d"(with_par(m0, par)),
               "d"(with_par(m1, par)), "d"(with_par(v0, par)), "d"(with_tag(v1, par, 0u)));
}

__device__ __forceinline__ bool rec_changed(const Raw& o, double m0, double m1, double v0, double v1) {
  return strip(o.a) != strip((unsigned long long)__double_as_longlong(m0)) ||
         strip(o.b) != strip((unsigned long long)__double_as_longlong(m1)) ||
         strip(o.c) != strip((unsigned long long)__double_as_longlong(v0)) ||
         strip2(o.d) != strip2((unsigned long long)__double_as_longlong(v1));
}

// --------------------------------------------------------------------------
// TMA staging of a CTA's slice of a level
// --------------------------------------------------------------------------
__device__ __forceinline__ void mbar_init(uint64_t* bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// this CTA's slice of level s: heads [a, b), entries [xa, xb) (host table,
// kept in shared memory for the first kSliceCap levels: no global round trip
// on the level-to-level chain)
constexpr int kSliceCap = 1024;
__device__ __forceinline__ int4 slice_of(const SLParams& P, const int4* s_slc, int s) {
  return s < kSliceCap ? s_slc[s] : __ldg(P.slice + size_t(s) * gridDim.x + blockIdx.x);
}
__device__ __forceinline__ void load_slices(const SLParams& P, int4* s_slc) {
  for (int s = threadIdx.x; s < min(P.num_sl, kSliceCap); s += blockDim.x)
    s_slc[s] = __ldg(P.slice + size_t(s) * gridDim.x + blockIdx.x);
}

struct HeadTopo {
  int32_t x0, nf, pin;
};

__device__ __forceinline__ HeadTopo load_topo(const SLParams& P, int h) {
  HeadTopo t;
  t.x0 = __ldg(P.hd_ptr + h);
  t.nf = __ldg(P.hd_ptr + h + 1) - t.x0;
  t.pin = __ldg(P.hd_pin + h);
  return t;
}

// forward stage: head rows and entry words of one CTA slice
constexpr int kFRowCap = 1024, kFEntCap = 2560;
// Per CTA: head rows and entry words of two levels (double-buffered, staged a
// level ahead; the arc records are read next to the source gathers), then the
// CTA's slice table.
struct FStageSet {
  int32_t ptr[2][kFRowCap + 8];
  int32_t pin[2][kFRowCap + 8];
  int32_t w[2][kFEntCap + 8];
  int32_t f[2][kFEntCap + 8];
  uint64_t full[2];
  int32_t ok[2];          // the slice fit the stage (else its heads read global)
};
constexpr size_t kFSlcOff = (sizeof(FStageSet) + 15) & ~size_t(15);   // int4 slice table after the stage
constexpr size_t kFStageBytes = kFSlcOff + sizeof(int4) * kSliceCap + sizeof(int32_t) * (kSliceCap + 4);

__device__ __forceinline__ bool fwd_fits(int a, int b, int xa, int xb) {
  return b > a && b - a <= kFRowCap && xb - xa <= kFEntCap;
}

// thread 0: stage rows and entry words of slice [a, b) (entries [xa, xb)) into buffer bf
__device__ __forceinline__ void fwd_issue(const SLParams& P, FStageSet* S, int bf, int a, int b, int xa, int xb) {
  const bool fits = fwd_fits(a, b, xa, xb);
  S->ok[bf] = fits ? 1 : 0;
  if (!fits) {
    mbar_arrive(&S->full[bf]);
    return;
  }
  const Window wp = window(a, b + 1, 4), wh = window(a, b, 4), wx = window(xa, xb, 4);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_expect_tx(&S->full[bf], wp.bytes + wh.bytes + 2 * wx.bytes);
  bulk_g2s(S->ptr[bf], P.hd_ptr + wp.start, wp.bytes, &S->full[bf]);
  bulk_g2s(S->pin[bf], P.hd_pin + wh.start, wh.bytes, &S->full[bf]);
  if (wx.bytes) {
    bulk_g2s(S->w[bf], P.ext_w + wx.start, wx.bytes, &S->full[bf]);
    bulk_g2s(S->f[bf], P.ext_f + wx.start, wx.bytes, &S->full[bf]);
  }
}

// L2 prefetch of a byte range (TMA bulk prefetch; 16-byte aligned, size a multiple of 16)
__device__ __forceinline__ void prefetch_l2(const void* p, uint32_t bytes) {
  if (bytes) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// the arc records of entries [xa, xb) (the next level's slice): off the dependency chain
__device__ __forceinline__ void sx_prefetch_rec(const SLParams& P, int xa, int xb) {
  if (xb <= xa) return;
  prefetch_l2(P.ext_ms + xa, uint32_t(xb - xa) * 16u);
  prefetch_l2(P.ext_fms + xa, uint32_t(xb - xa) * 16u);
}

// Folded pin p (fold.cpp) on its single fanin arc e' = (j -> p) (word f,
// record fms, entry x): merge1, the nf = 1 merge (bit-identical to merge_rf),
// on j's words rj.  Returns p's words as a store would leave them (parity
// LSB), which is what its sink reads.  A non-unate e' has two candidates: its
// arg-max / weights are stored per entry for the backward.
template <bool kLSE>
__device__ __forceinline__ Raw sl_fold(const SLParams& P, int32_t f, const float4& fms, int x, const Raw& rj) {
  const int u2 = int(uint32_t(f) >> kUnateShift);
  Merge1 m;
  merge1<kLSE>(unpack(rj), u2, fms, double(P.n_sigma), double(P.tau), P.inv_tau, m);
  if (P.store_fold) {
    st_state(P.state + (f & kSrcMask), m.mu[0], m.mu[1], m.var[0], m.var[1], P.par);
    if (!kLSE) P.win[f & kSrcMask] = m.win;
    else P.wts[__ldg(P.ext_fq + x)] = m.wt;
  }
  if (u2 == 2) {
    if (!kLSE) {
      if (P.elog) {   // eval_kernel: record the word this cone pass overwrites
        const int32_t o = P.fwin[x];
        if (o != m.win) {
          const uint32_t k = atomicAdd(P.elog_n + 1, 1u);
          if (k < uint32_t(P.elog_cap)) P.flog[k] = make_int2(x, o);
        }
      }
      P.fwin[x] = m.win;
    } else {
      P.efw[x] = m.wt;
    }
  }
  return m.stored(P.par);
}

// cone pass: super-levels that may hold a dirty head, per CTA in shared
// memory (flushed to sl_cnt once per level).  Bit 0 (s_mark): a head of the
// level was stamped dirty; bit 1 (s_mark + kMarkWords): a source with a long
// consumer row changed -- the level's heads with such a source check it.
constexpr int kMarkWords = 64;   // levels >= 32 * kMarkWords are flagged in global directly

// (read before the atomic: most marks find the bit set already -- the heads of a level mark the
// same few levels, and same-word shared atomics serialize: ncu / trace, ~20 us per level at C3 1 %)
__device__ __forceinline__ void mark_level(const SLParams& P, uint32_t* s_mark, int s, uint32_t kind) {
  if (s < 32 * kMarkWords) {
    uint32_t* w = s_mark + (kind - 1) * kMarkWords + (s >> 5);
    const uint32_t b = 1u << (s & 31);
    if (!(*reinterpret_cast<volatile uint32_t*>(w) & b)) atomicOr(w, b);
  } else if (!(__ldcg(P.sl_cnt + s) & kind)) {
    atomicOr(P.sl_cnt + s, kind);
  }
}

// flag levels [lo, hi] (kind 2)
__device__ __forceinline__ void mark_range(const SLParams& P, uint32_t* s_mark, int lo, int hi) {
  for (int w = lo >> 5; w <= (hi >> 5); ++w) {
    if (w >= kMarkWords) {
      for (int s = max(lo, 32 * w); s <= hi; ++s) atomicOr(P.sl_cnt + s, 2u);
      return;
    }
    uint32_t m = 0xffffffffu;
    if (w == (lo >> 5)) m &= 0xffffffffu << (lo & 31);
    if (w == (hi >> 5)) m &= 0xffffffffu >> (31 - (hi & 31));
    if ((*reinterpret_cast<volatile uint32_t*>(s_mark + kMarkWords + w) & m) != m) atomicOr(s_mark + kMarkWords + w, m);
  }
}

// super-level of head q: last s with sl_ptr[s] <= q (level table in shared memory)
__device__ __forceinline__ int sl_of(const SLParams& P, const int32_t* s_slp, int q) {
  int lo = 0, hi = P.num_sl;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    const int v = mid <= kSliceCap ? s_slp[mid] : __ldg(P.sl_ptr + mid);
    if (v <= q) lo = mid;
    else hi = mid;
  }
  return lo;
}

// where a head's entry words and arc records are read: its staged slice
// (shared memory) or global
struct EntSrc {
  const int32_t* w;
  const int32_t* f;
  const float4* ms;
  const float4* fms;
  const Raw* gath;   // gathered source records (shared memory) or nullptr: gather here
};

// Merge of a head with exactly NF entries (compile-time: no predication on the
// entry count; heads of a super-level are ordered by shape, fold.cpp, so a
// warp's heads take the same path).  Entry words from `ws` / `fs` (staged in
// shared memory, or global), arc records from global.  Returns the pins
// evaluated (the head and its folded input pins).
template <bool kLSE, int NF>
__device__ __forceinline__ int sl_fwd_core(const SLParams& P, const HeadTopo& t, const EntSrc& E, RfOut& R, RfOut& F,
                                           unsigned long long* ph) {
  const double ns = double(P.n_sigma);
  int npins = 1;
  int32_t w[NF], f[NF];
  float4 ms[NF], fms[NF];
  Raw r[NF];
#pragma unroll
  for (int k = 0; k < NF; ++k) w[k] = E.w[k];
#pragma unroll
  for (int k = 0; k < NF; ++k)   // the dependent gathers (already landed in shared memory, or issued here)
    r[k] = E.gath ? E.gath[k] : ld_raw(P.state + (w[k] & kSrcMask));
  // everything else is independent of the chain: issued before any use
#pragma unroll
  for (int k = 0; k < NF; ++k) {
    ms[k] = E.ms[k];
    if ((w[k] >> kFoldBit) & 1) {
      f[k] = E.f[k];
      fms[k] = E.fms[k];
    }
  }
#ifdef INSTA_SL_PHASES
  if (ph && !ph[4]) {   // debug: the first head's gathers and records have landed
    const unsigned long long dep = (r[0].a | __float_as_uint(ms[NF - 1].x)) & 0ull;
    ph[4] = gtimer() + dep;
  }
#endif
#pragma unroll
  for (int k = 0; k < NF; ++k) {
    if ((w[k] >> kFoldBit) & 1) {
      r[k] = sl_fold<kLSE>(P, f[k], fms[k], t.x0 + k, r[k]);
      ++npins;
    }
  }
  auto arc = [&](int k, int32_t& w_, float4& ms_, Raw& r_) {
    w_ = w[k];
    ms_ = ms[k];
    r_ = r[k];
  };
  R = merge_rf_unrolled<kLSE, NF>(ns, double(P.tau), P.inv_tau, 0, NF, arc);
  F = merge_rf_unrolled<kLSE, NF>(ns, double(P.tau), P.inv_tau, 1, NF, arc);
  if (kLSE) {
#pragma unroll
    for (int k = 0; k < NF; ++k) {
      const float2 wr = arc_weights(ns, P.inv_tau, 0, k, R, arc);
      const float2 wf = arc_weights(ns, P.inv_tau, 1, k, F, arc);
      P.ew[t.x0 + k] = make_float4(wr.x, wr.y, wf.x, wf.y);
    }
  }
  return npins;
}

// wide head (not in netlist-shaped graphs): folded pins once, then the
// generic merge re-reading its entries from global (the same words)
template <bool kLSE>
__device__ __noinline__ int sl_fwd_wide(const SLParams P, const HeadTopo t, RfOut& R, RfOut& F) {
  const double ns = double(P.n_sigma);
  int npins = 1;
  for (int k = 0; k < t.nf; ++k) {
    const int32_t w = __ldg(P.ext_w + t.x0 + k);
    if ((w >> kFoldBit) & 1) {
      (void)sl_fold<kLSE>(P, __ldg(P.ext_f + t.x0 + k), P.ext_fms[t.x0 + k], t.x0 + k,
                          ld_raw(P.state + (w & kSrcMask)));
      ++npins;
    }
  }
  auto arc = [&](int k, int32_t& w_, float4& ms_, Raw& r_) {
    w_ = __ldg(P.ext_w + t.x0 + k);
    ms_ = P.ext_ms[t.x0 + k];
    r_ = ld_raw(P.state + (w_ & kSrcMask));
    if ((w_ >> kFoldBit) & 1) {
      const int32_t f = __ldg(P.ext_f + t.x0 + k);
      Merge1 m;
      merge1<kLSE>(unpack(r_), int(uint32_t(f) >> kUnateShift), P.ext_fms[t.x0 + k], ns, double(P.tau), P.inv_tau,
                   m);
      r_ = m.stored(P.par);
    }
  };
  R = merge_rf<kLSE>(ns, double(P.tau), P.inv_tau, 0, t.nf, arc);
  F = merge_rf<kLSE>(ns, double(P.tau), P.inv_tau, 1, t.nf, arc);
  if (kLSE) {
    for (int k = 0; k < t.nf; ++k) {
      const float2 wr = arc_weights(ns, P.inv_tau, 0, k, R, arc);
      const float2 wf = arc_weights(ns, P.inv_tau, 1, k, F, arc);
      P.ew[t.x0 + k] = make_float4(wr.x, wr.y, wf.x, wf.y);
    }
  }
  return npins;
}

// Forward of one head (both rf).  kInc: compare with the previous record and,
// when it changed, mark the consumer heads.  Returns the pins evaluated.
template <bool kLSE, bool kInc>
__device__ __forceinline__ int sl_fwd_head(const SLParams& P, int h, const HeadTopo& t, const EntSrc& E,
                                           uint32_t* s_mark, const int32_t* s_slp, uint32_t stamp,
                                           unsigned long long* ph = nullptr) {
  RfOut R, F;
  Raw old;
  if (kInc) old = ld_raw(P.state + t.pin);
  int npins;
  switch (t.nf) {
    case 1: npins = sl_fwd_core<kLSE, 1>(P, t, E, R, F, ph); break;
    case 2: npins = sl_fwd_core<kLSE, 2>(P, t, E, R, F, ph); break;
    case 3: npins = sl_fwd_core<kLSE, 3>(P, t, E, R, F, ph); break;
    case 4: npins = sl_fwd_core<kLSE, 4>(P, t, E, R, F, ph); break;
    default: npins = sl_fwd_wide<kLSE>(P, t, R, F); break;
  }
  if (!kLSE) {
    const int32_t nw = R.win | (F.win << 16);
    if (kInc && P.elog) {   // eval_kernel: record what this cone pass overwrites (undo log)
      const int32_t ow = P.hwin[h];
      if (ow != nw || rec_changed(old, R.mu, F.mu, R.var, F.var)) {
        const uint32_t k = atomicAdd(P.elog_n, 1u);
        if (k < uint32_t(P.elog_cap)) {
          EvLog e;
          e.rec = old;
          e.pin = t.pin;
          e.h = h;
          e.win = ow;
          e.pad = 0;
          P.elog[k] = e;
        }
      }
    }
    P.hwin[h] = nw;
  }
  if (kInc && P.btouch) P.btouch[h] = P.bepoch;   // its arg-max / weights may differ from the backward snapshot
  if (kInc) {
    if (rec_changed(old, R.mu, F.mu, R.var, F.var)) {
      st_state(P.state + t.pin, R.mu, F.mu, R.var, F.var, P.par);
      // consumers (later levels): a short row is stamped dirty one by one; a
      // long row's consumers see the change through chg (levels flagged)
      P.chg[t.pin] = stamp;
      if (P.ep_blk) {   // an endpoint: its slack block is recomputed after the pass
        const int k = __ldg(P.hd_eop + h);
        if (k >= 0) {
          const int b = (k / kRedThreads) % P.slack_nb;
          // (read first: a few words take every endpoint's flag, global atomics on them serialize)
          if (!((__ldcg(P.ep_blk + (b >> 5)) >> (b & 31)) & 1u)) atomicOr(P.ep_blk + (b >> 5), 1u << (b & 31));
        }
      }
      const int r0 = __ldg(P.hfo_ptr + h), r1 = __ldg(P.hfo_ptr + h + 1);
      if (r1 - r0 <= kConeRow) {
        for (int r = r0; r < r1; r += 8) {   // the row's loads in flight together
          int32_t q[8], lv[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            q[j] = r + j < r1 ? __ldg(P.hfo + r + j) : -1;
            lv[j] = r + j < r1 ? __ldg(P.hfo_sl + r + j) : 0;
          }
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            if (q[j] >= 0) {
              P.dirty[q[j]] = stamp;
              mark_level(P, s_mark, lv[j], 1u);
            }
          }
        }
      } else {
        const int32_t cs = __ldg(P.hd_csl + h);
        mark_range(P, s_mark, cs & 0xffff, int(uint32_t(cs) >> 16));
      }
    }
  } else {
    st_state(P.state + t.pin, R.mu, F.mu, R.var, F.var, P.par);
  }
  return npins;
}


// Cone pass (kInc): is head h dirty?  Stamped by insta_update_arcs (an arc it
// evaluates changed) or one of its entries' source records changed in this
// pass (chg, written by the recomputed source head before the level barrier).
__device__ __forceinline__ bool head_dirty(const SLParams& P, int h, const int32_t* w, int nf, uint32_t lvl,
                                           uint32_t stamp) {
  if (__ldcg(P.dirty + h) == stamp) return true;
  if (!(lvl & 2u) || !__ldg(P.hd_hsrc + h)) return false;
  uint32_t c[4];   // every load in flight at once
#pragma unroll
  for (int k = 0; k < 4; ++k) c[k] = k < nf ? __ldcg(P.chg + (w[k] & kSrcMask)) : 0u;
  bool any = false;
#pragma unroll
  for (int k = 0; k < 4; ++k) any |= c[k] == stamp;
  for (int k = 4; k < nf && !any; ++k) any = __ldcg(P.chg + (w[k] & kSrcMask)) == stamp;
  return any;
}

// flush the CTA's level flags (after a CTA barrier; before the grid barrier):
// each (level, kind) flag is published at most once per pass by a CTA (s_pub)
__device__ __forceinline__ void mark_flush(const SLParams& P, uint32_t* s_mark, uint32_t* s_pub) {
  for (int k = threadIdx.x; k < 2 * kMarkWords; k += blockDim.x) {
    uint32_t m = s_mark[k] & ~s_pub[k];
    s_mark[k] = 0u;
    s_pub[k] |= m;
    const uint32_t kind = k < kMarkWords ? 1u : 2u;
    const int w = k % kMarkWords;
    while (m) {
      const int b = __ffs(m) - 1;
      m &= m - 1;
      const int sl = 32 * w + b;
      if (sl < P.num_sl) atomicOr(P.sl_cnt + sl, kind);
    }
  }
}

// Shared memory of a cone pass that reads topology from global (small cone).
struct ConeSm {
  uint32_t mark[2 * kMarkWords];
  uint32_t pub[2 * kMarkWords];
  uint32_t cnt;
  int32_t next;
};

// Unstaged cone pass over levels 1 .. L-1 (flags in P.sl_cnt, dirty stamps ==
// stamp): jumps from flagged level to flagged level -- every flag at or past
// the current level is final (the levels before it are done) -- with one grid
// barrier per level that recomputed something.  The caller has zeroed
// cs.pub, and barriers the grid before and after.
template <bool kLSE>
__device__ __forceinline__ void cone_levels(const SLParams& P, uint32_t stamp, ConeSm& cs, const int4* s_slc,
                                            const int32_t* s_slp, uint32_t& nbar, uint32_t& nrec) {
  const int tid = threadIdx.x, L = P.num_sl;
  bool need_bar = false;
  for (int s = 1; s < L; ++s) {
    if (need_bar) grid_sync(P.bar, ++nbar, P.trace);
    need_bar = false;
    if (tid < 32) {   // one warp scans the flags 32 at a time
      int nx = L;
      for (int base = s; base < L; base += 32) {
        const uint32_t f = base + tid < L ? __ldcg(P.sl_cnt + base + tid) : 0u;
        const uint32_t hit = __ballot_sync(0xffffffffu, f != 0u);
        if (hit) {
          nx = base + __ffs(hit) - 1;
          const uint32_t fv = __shfl_sync(0xffffffffu, f, __ffs(hit) - 1);
          if (tid == 0) cs.cnt = fv;
          break;
        }
      }
      if (tid == 0) cs.next = nx;
    }
    __syncthreads();
    s = cs.next;
    const uint32_t lvl = cs.cnt;
    __syncthreads();
    if (s >= L) break;
    need_bar = true;
    const int4 sc = slice_of(P, s_slc, s);
    for (int h = sc.x + tid; h < sc.y; h += blockDim.x) {
      const HeadTopo t = load_topo(P, h);
      const EntSrc E{P.ext_w + t.x0, P.ext_f + t.x0, P.ext_ms + t.x0, P.ext_fms + t.x0, nullptr};
      if (!head_dirty(P, h, E.w, t.nf, lvl, stamp)) continue;
      nrec += uint32_t(sl_fwd_head<kLSE, true>(P, h, t, E, cs.mark, s_slp, stamp));
    }
    __syncthreads();
    mark_flush(P, cs.mark, cs.pub);
  }
}

// kMode 0: full pass.  1: cone pass over the staged slices (large updates).
// 2: cone pass reading only the dirty heads' topology (small updates).  The
// cone passes recompute dirty heads only and skip (without a barrier) every
// level no head flagged: its flag is final once the levels before it are done.
template <bool kLSE, int kMode>
__global__ void __launch_bounds__(kSLFwdThreads, 1) fwdl_kernel(SLParams P) {
  constexpr bool kInc = kMode != 0;
  extern __shared__ __align__(128) unsigned char sl_smem[];
  __shared__ ConeSm cs;
  const int gt = blockIdx.x * blockDim.x + threadIdx.x;
  const int nthr = gridDim.x * blockDim.x;
  const int tid = threadIdx.x;
  const int L = P.num_sl;
  uint32_t nbar = 0, nrec = 0;
  if (P.trace && gt == 0) P.trace[0] = gtimer();
  for (int k = tid; k < 2 * kMarkWords; k += blockDim.x) cs.mark[k] = cs.pub[k] = 0u;
  FStageSet* S = reinterpret_cast<FStageSet*>(sl_smem);
  int4* s_slc = reinterpret_cast<int4*>(sl_smem + kFSlcOff);
  int32_t* s_slp = reinterpret_cast<int32_t*>(s_slc + kSliceCap);   // level table (cone: level of a head)
  load_slices(P, s_slc);
  for (int v = tid; v <= min(P.num_sl, kSliceCap); v += blockDim.x) s_slp[v] = __ldg(P.sl_ptr + v);
  __syncthreads();
  if constexpr (kMode == 2) {
    cone_levels<kLSE>(P, P.stamp, cs, s_slc, s_slp, nbar, nrec);
  } else {
    if (tid == 0) {
      mbar_init(&S->full[0]);
      mbar_init(&S->full[1]);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      if (L > 1) {
        const int4 c = slice_of(P, s_slc, 1);
        fwd_issue(P, S, 1, c.x, c.y, c.z, c.w);
      }
    }
    if (!kInc) {
      for (int s = gt; s < L; s += nthr) P.sl_cnt[s] = 0u;   // a full pass supersedes pending flags
      // startpoints: clock arrival distribution, mean and variance per rf
      for (int i = gt; i < P.num_src; i += nthr) {
        const float4 v = __ldg(P.src_ms + i);
        st_state(P.state + i, double(v.x), double(v.y), double(v.z) * double(v.z), double(v.w) * double(v.w), P.par);
      }
    }
    uint32_t phase[2] = {0u, 0u};
    bool need_bar = !kInc;   // cone: flags of level 1 come from insta_update_arcs (an earlier launch)
    for (int s = 1; s < L; ++s) {
      const int bf = s & 1;
      __syncthreads();   // every thread is done with level s - 1 (rows buffer bf ^ 1)
      if (tid == 0 && s + 1 < L) {   // rows and entry words of level s + 1
        const int4 c = slice_of(P, s_slc, s + 1);
        fwd_issue(P, S, bf ^ 1, c.x, c.y, c.z, c.w);
        if (kInc) sx_prefetch_rec(P, c.z, c.w);   // and its arc records to L2 (off the dirty heads' chain)
      }
      if (need_bar) grid_sync(P.bar, ++nbar, P.trace);   // levels < s are complete
      unsigned long long* ph = nullptr;
#ifdef INSTA_SL_PHASES
      if (P.trace && tid == 0) {   // debug: per (level, CTA) timestamps
        ph = P.trace + 512 + size_t(L + 8) * 2 * gridDim.x + (size_t(s) * gridDim.x + blockIdx.x) * 8;
        ph[0] = gtimer();
      }
#endif
      bool work = true;
      uint32_t lvl = 0;
      if (kInc) {   // flags of level s come from levels < s: final here
        if (tid == 0) cs.cnt = __ldcg(P.sl_cnt + s);
        __syncthreads();
        lvl = cs.cnt;
        work = lvl != 0;
        need_bar = work;
#ifdef INSTA_SL_PHASES
        if (ph) ph[1] = gtimer();
#endif
      }
      const int4 sc = slice_of(P, s_slc, s);
      const int a = sc.x, b = sc.y;
      mbar_wait(&S->full[bf], phase[bf]);
      phase[bf] ^= 1u;
      const bool ok = S->ok[bf] != 0;
#ifdef INSTA_SL_PHASES
      if (ph) ph[2] = gtimer();
#endif
      if (!work) continue;
      const Window wp = window(a, b + 1, 4), wh = window(a, b, 4);
      const int xa = sc.z;
      const Window wx = window(xa, sc.w, 4);
      for (int h = a + tid; h < b; h += blockDim.x) {
        const int r = h - a;
        HeadTopo t;
        EntSrc E;   // entry words, arc records: staged slice, or global
        if (ok) {
          t.x0 = S->ptr[bf][wp.off + r];
          t.nf = S->ptr[bf][wp.off + r + 1] - t.x0;
          t.pin = S->pin[bf][wh.off + r];
          const int xr = wx.off + t.x0 - xa;
          E = EntSrc{S->w[bf] + xr, S->f[bf] + xr, P.ext_ms + t.x0, P.ext_fms + t.x0, nullptr};
        } else {
          t = load_topo(P, h);
          E = EntSrc{P.ext_w + t.x0, P.ext_f + t.x0, P.ext_ms + t.x0, P.ext_fms + t.x0, nullptr};
        }
        if (kInc) {
          if (!head_dirty(P, h, E.w, t.nf, lvl, P.stamp)) continue;
#ifdef INSTA_SL_PHASES
          if (ph && !ph[3]) ph[3] = gtimer();   // debug: the first dirty head found
#endif
          nrec += uint32_t(sl_fwd_head<kLSE, true>(P, h, t, E, cs.mark, s_slp, P.stamp, ph));
#ifdef INSTA_SL_PHASES
          if (ph && !ph[7]) ph[7] = gtimer();   // debug: its recompute and marks done
#endif
        } else {
          (void)sl_fwd_head<kLSE, false>(P, h, t, E, cs.mark, s_slp, P.stamp, ph);
        }
      }
#ifdef INSTA_SL_PHASES
      if (ph) ph[5] = gtimer();
#endif
      if (kInc) {
        __syncthreads();
        mark_flush(P, cs.mark, cs.pub);
#ifdef INSTA_SL_PHASES
        if (ph) ph[6] = gtimer();
#endif
      }
    }
  }
  if (kInc) {
    // clear the level flags for the next cone pass (every CTA has read them)
    grid_sync(P.bar, ++nbar, P.trace);
    for (int s = gt; s < L; s += nthr) P.sl_cnt[s] = 0u;
    const uint32_t n = __reduce_add_sync(0xffffffffu, nrec);
    if ((tid & 31) == 0 && n) atomicAdd(P.counters, (unsigned long long)n);
  }
  grid_exit(P.bar);
}

// --------------------------------------------------------------------------
// Entry-parallel forward (fwdx_kernel; the default full pass).
//
// fwdl_kernel runs a head's whole merge on one thread: the gathers, every
// folded pin (merge1) and every candidate of both transitions form one serial
// chain of ~600 instructions, which (ncu: 12 warps / SM, 27 cycles per issued
// instruction, 60 % of the samples in the CTA barrier waiting for the slowest
// thread) is what a level costs.  Here a level is two short phases:
//   (1) entry phase, a thread per entry: gather the source record, evaluate the
//       folded pin (merge1), form both transitions' candidates (Eq 1-3) and
//       reduce a non-unate arc's pair (strict ">": the second replaces the first
//       only if greater), into a shared-memory slot {A0, A1, mu, var} per rf;
//   (2) head phase, a thread per head: the first arg-max over its entries' slots
//       in fanin order (strict ">", Alg 2 l.4 / P:L97), the LSE normalizer in
//       candidate order (Eq 4), the store and the Eq 6 weights.
// The candidate values are those of make_cand, the arg-max is the one of the
// sequential scan (a pair pre-reduced with strict ">" then compared with strict
// ">" selects the same first maximum), the sums run in the same order: the
// arrivals, arg-max words and weights equal fwdl_kernel's bit for bit.
// kFlow: no grid barrier -- a gather re-polls a record until its parity is this
// pass's (the dataflow synchronization of schedule 2); the CTA barriers between
// the phases and levels stay (they order the shared stage only).
// --------------------------------------------------------------------------
// threads per CTA (one CTA per SM): hard mode 768 (<= 80 registers), LSE 512 (its
// exponentials and weights need more registers; measured best of 384-768 at C4)
#ifndef INSTA_SX_THREADS
#define INSTA_SX_THREADS 768
#endif
#ifndef INSTA_SX_THREADS_LSE
#define INSTA_SX_THREADS_LSE 512
#endif
constexpr int kSXThreads = INSTA_SX_THREADS;
constexpr int kSXThreadsLSE = INSTA_SX_THREADS_LSE;
__host__ __device__ constexpr int sx_threads(bool lse) { return lse ? kSXThreadsLSE : kSXThreads; }
constexpr int kXCap = 2048;   // entries of a slice held in shared memory
#ifndef INSTA_SX_PREFETCH
#define INSTA_SX_PREFETCH 1
#endif
constexpr bool kSXPrefetch = INSTA_SX_PREFETCH != 0;   // L2 prefetch of a later level's arc records
#ifndef INSTA_SX_AHEAD
#define INSTA_SX_AHEAD 1
#endif
constexpr int kSXAhead = INSTA_SX_AHEAD;               // how many levels ahead
// head merge specialized for 1-4 entries: LSE only (measured: hard mode is faster with the generic loop)
#ifndef INSTA_SX_HEADN
#define INSTA_SX_HEADN 2
#endif
template <bool kLSE>
__device__ __forceinline__ constexpr bool sx_headn() { return INSTA_SX_HEADN == 1 || (INSTA_SX_HEADN == 2 && kLSE); }
struct XCand {
  double A0, A1, mu, var;     // corners of the s0 / non-unate second candidate; the pair's winner
};
constexpr size_t kXOff = (kFStageBytes + 127) & ~size_t(127);
constexpr size_t kXStageBytes = kXOff + sizeof(XCand) * 2 * kXCap + kXCap;

template <bool kFlow>
__device__ __forceinline__ void sx_await(const SLParams& P, int j, Raw& r) {
  if (!kFlow) return;
  uint32_t n = 0;
  while (!raw_ready(r, P.par)) {
    if (++n > (1u << 23)) __trap();   // bounded: never a silent hang
    r = ld_raw(P.state + j);
  }
}

// entry x (slot of the slice): folded pin, candidates of both transitions
template <bool kLSE>
__device__ __forceinline__ void sx_entry(const SLParams& P, int x, int32_t w, int32_t f, const float4& ms,
                                         const float4& fms, Raw r, XCand* xc, uint8_t* xs) {
  if ((w >> kFoldBit) & 1) r = sl_fold<kLSE>(P, f, fms, x, r);
  const Gath st = unpack(r);
  const int u = int(uint32_t(w) >> kUnateShift);
  const double ns = double(P.n_sigma);
  uint32_t sb = 0u;
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    const Cand c0 = make_cand(st, ms, rf, src_tr(rf, u, 0), ns);
    XCand o;
    o.A0 = c0.A;
    o.A1 = c0.A;
    o.mu = c0.mu;
    o.var = c0.var;
    if (u == 2) {
      const Cand c1 = make_cand(st, ms, rf, rf ^ 1, ns);
      o.A1 = c1.A;
      if (c1.A > c0.A) {   // strict: s = rf wins ties (merge_rf order)
        o.mu = c1.mu;
        o.var = c1.var;
        sb |= 1u << rf;
      }
    }
    xc[rf] = o;
  }
  *xs = uint8_t(sb);
}

// head h with exactly NF entries (compile-time: every slot load is issued before
// the scan; heads of a slice are ordered by shape, fold.cpp, so a warp's heads
// take the same case).  The same operations in the same order as sx_head.
template <bool kLSE, int NF>
__device__ __forceinline__ void sx_head_n(const SLParams& P, int h, int x0, int pin, const int32_t* w,
                                          const XCand* xc, const uint8_t* xs) {
  const double ns = double(P.n_sigma);
  XCand c[NF][2];
  uint32_t sb[NF];
  int u[NF];
#pragma unroll
  for (int k = 0; k < NF; ++k) {
    sb[k] = xs[k];
    u[k] = int(uint32_t(w[k]) >> kUnateShift);
    c[k][0] = xc[2 * k];
    c[k][1] = xc[2 * k + 1];
  }
  double mu[2], var[2], best[2];
  float sum[2];
  int win[2];
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    double b = ((sb[0] >> rf) & 1u) ? c[0][rf].A1 : c[0][rf].A0;
    int bk = 0;
    double bm = c[0][rf].mu, bv = c[0][rf].var;
#pragma unroll
    for (int k = 1; k < NF; ++k) {
      const double A = ((sb[k] >> rf) & 1u) ? c[k][rf].A1 : c[k][rf].A0;
      if (A > b) {   // Alg 2 l.4: replace only if strictly greater
        b = A;
        bk = k;
        bm = c[k][rf].mu;
        bv = c[k][rf].var;
      }
    }
    int uw = u[0];
    uint32_t sbw = sb[0];
#pragma unroll
    for (int k = 1; k < NF; ++k)
      if (bk == k) {
        uw = u[k];
        sbw = sb[k];
      }
    const int sw = ((sbw >> rf) & 1u) ? (rf ^ 1) : src_tr(rf, uw, 0);
    mu[rf] = bm;
    var[rf] = bv;
    best[rf] = b;
    win[rf] = bk | (sw << 15);
    sum[rf] = 0.f;
    if (kLSE) {
      float s = 0.f;
#pragma unroll
      for (int k = 0; k < NF; ++k) {
        s += lse_w(c[k][rf].A0, b, P.inv_tau);
        if (u[k] == 2) s += lse_w(c[k][rf].A1, b, P.inv_tau);
      }
      sum[rf] = s;
      mu[rf] = lse_arrival(b, double(P.tau), s) - ns * double(sigma_of(bv));
    }
  }
  st_state(P.state + pin, mu[0], mu[1], var[0], var[1], P.par);
  if (!kLSE) {
    P.hwin[h] = win[0] | (win[1] << 16);
  } else {
    const float inv0 = 1.f / sum[0], inv1 = 1.f / sum[1];
#pragma unroll
    for (int k = 0; k < NF; ++k) {
      float wt[2][2] = {{0.f, 0.f}, {0.f, 0.f}};
#pragma unroll
      for (int rf = 0; rf < 2; ++rf) {
        const float inv = rf ? inv1 : inv0;
        wt[rf][src_tr(rf, u[k], 0)] = lse_w(c[k][rf].A0, best[rf], P.inv_tau) * inv;
        if (u[k] == 2) wt[rf][rf ^ 1] = lse_w(c[k][rf].A1, best[rf], P.inv_tau) * inv;
      }
      P.ew[x0 + k] = make_float4(wt[0][0], wt[0][1], wt[1][0], wt[1][1]);
    }
  }
}

// head h with entries [x0, x0 + nf): words w[k], slots xc[2k + rf], pair bits xs[k]
template <bool kLSE>
__device__ __forceinline__ void sx_head(const SLParams& P, int h, int x0, int nf, int pin, const int32_t* w,
                                        const XCand* xc, const uint8_t* xs) {
  const double ns = double(P.n_sigma);
  double mu[2], var[2], best[2];
  float sum[2];
  int win[2];
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    double b = 0.0;
    int bk = 0;
    for (int k = 0; k < nf; ++k) {
      const XCand& c = xc[2 * k + rf];
      const double A = ((xs[k] >> rf) & 1u) ? c.A1 : c.A0;
      if (k == 0 || A > b) {   // Alg 2 l.4: replace only if strictly greater
        b = A;
        bk = k;
      }
    }
    const XCand& cw = xc[2 * bk + rf];
    const int uw = int(uint32_t(w[bk]) >> kUnateShift);
    const int sw = ((xs[bk] >> rf) & 1u) ? (rf ^ 1) : src_tr(rf, uw, 0);
    mu[rf] = cw.mu;
    var[rf] = cw.var;
    best[rf] = b;
    win[rf] = bk | (sw << 15);
    sum[rf] = 0.f;
    if (kLSE) {   // Eq 4 over the candidates in merge order; reading R1 for sigma
      float s = 0.f;
      for (int k = 0; k < nf; ++k) {
        s += lse_w(xc[2 * k + rf].A0, b, P.inv_tau);
        if ((uint32_t(w[k]) >> kUnateShift) == 2u) s += lse_w(xc[2 * k + rf].A1, b, P.inv_tau);
      }
      sum[rf] = s;
      mu[rf] = lse_arrival(b, double(P.tau), s) - ns * double(sigma_of(cw.var));
    }
  }
  st_state(P.state + pin, mu[0], mu[1], var[0], var[1], P.par);
  if (!kLSE) {
    P.hwin[h] = win[0] | (win[1] << 16);
  } else {
    const float inv0 = 1.f / sum[0], inv1 = 1.f / sum[1];
    for (int k = 0; k < nf; ++k) {   // Eq 6 weights (arc_weights)
      const int u = int(uint32_t(w[k]) >> kUnateShift);
      float wt[2][2] = {{0.f, 0.f}, {0.f, 0.f}};
#pragma unroll
      for (int rf = 0; rf < 2; ++rf) {
        const float inv = rf ? inv1 : inv0;
        wt[rf][src_tr(rf, u, 0)] = lse_w(xc[2 * k + rf].A0, best[rf], P.inv_tau) * inv;
        if (u == 2) wt[rf][rf ^ 1] = lse_w(xc[2 * k + rf].A1, best[rf], P.inv_tau) * inv;
      }
      P.ew[x0 + k] = make_float4(wt[0][0], wt[0][1], wt[1][0], wt[1][1]);
    }
  }
}

// one level of fwdx_kernel: (1) entry phase, CTA barrier, (2) head phase.  xc / xs are indexed by entry
// id (shared memory, or the CTA's global buffer for a slice beyond kXCap entries).
template <bool kLSE, bool kFlow>
__device__ __forceinline__ void sx_level(const SLParams& P, int a, int b, int xa, int xb, const int32_t* Pt,
                                         const int32_t* Pn, const int32_t* Wx, const int32_t* Fx, XCand* xc,
                                         uint8_t* xs, unsigned long long* ph) {
  const int tid = threadIdx.x, nt = blockDim.x;
  // (1) entries: two per thread in flight (loads of both issued before either is used)
  for (int x = xa + tid; x < xb; x += 2 * nt) {
    const int y = x + nt;
    const bool two = y < xb;
    const int32_t w0 = Wx[x], w1 = two ? Wx[y] : 0;
    const float4 m0 = P.ext_ms[x];
    const float4 m1 = two ? P.ext_ms[y] : make_float4(0.f, 0.f, 0.f, 0.f);
    const bool f0 = (w0 >> kFoldBit) & 1, f1 = two && ((w1 >> kFoldBit) & 1);
    const int32_t g0 = f0 ? Fx[x] : 0, g1 = f1 ? Fx[y] : 0;
    const float4 n0 = f0 ? P.ext_fms[x] : m0;
    const float4 n1 = f1 ? P.ext_fms[y] : m1;
    Raw r0 = ld_raw(P.state + (w0 & kSrcMask));
    Raw r1;
    if (two) r1 = ld_raw(P.state + (w1 & kSrcMask));
    sx_await<kFlow>(P, w0 & kSrcMask, r0);
#ifdef INSTA_SL_PHASES
    if (ph && x == xa) ph[4] = gtimer() + ((r0.a | __float_as_uint(m0.x)) & 0ull);
#endif
    sx_entry<kLSE>(P, x, w0, g0, m0, n0, r0, xc + 2 * x, xs + x);
    if (two) {
      sx_await<kFlow>(P, w1 & kSrcMask, r1);
      sx_entry<kLSE>(P, y, w1, g1, m1, n1, r1, xc + 2 * y, xs + y);
    }
  }
  __syncthreads();
#ifdef INSTA_SL_PHASES
  if (ph) ph[6] = gtimer();   // debug: every entry of the CTA's slice done
#endif
  // (2) heads
  for (int h = a + tid; h < b; h += nt) {
    const int x0 = Pt[h], nf = Pt[h + 1] - x0;
    switch (sx_headn<kLSE>() ? nf : 0) {
      case 1: sx_head_n<kLSE, 1>(P, h, x0, Pn[h], Wx + x0, xc + 2 * x0, xs + x0); break;
      case 2: sx_head_n<kLSE, 2>(P, h, x0, Pn[h], Wx + x0, xc + 2 * x0, xs + x0); break;
      case 3: sx_head_n<kLSE, 3>(P, h, x0, Pn[h], Wx + x0, xc + 2 * x0, xs + x0); break;
      case 4: sx_head_n<kLSE, 4>(P, h, x0, Pn[h], Wx + x0, xc + 2 * x0, xs + x0); break;
      default: sx_head<kLSE>(P, h, x0, nf, Pn[h], Wx + x0, xc + 2 * x0, xs + x0); break;
    }
  }
}

template <bool kLSE, bool kFlow>
__global__ void __launch_bounds__(sx_threads(kLSE), 1) fwdx_kernel(SLParams P) {
  extern __shared__ __align__(128) unsigned char sl_smem[];
  const int gt = blockIdx.x * blockDim.x + threadIdx.x;
  const int nthr = gridDim.x * blockDim.x;
  const int tid = threadIdx.x;
  const int L = P.num_sl;
  FStageSet* S = reinterpret_cast<FStageSet*>(sl_smem);
  int4* s_slc = reinterpret_cast<int4*>(sl_smem + kFSlcOff);
  XCand* xc_s = reinterpret_cast<XCand*>(sl_smem + kXOff);
  uint8_t* xs_s = reinterpret_cast<uint8_t*>(xc_s + 2 * kXCap);
  XCand* xc_g = P.xscr ? reinterpret_cast<XCand*>(P.xscr) + size_t(blockIdx.x) * 2 * P.xscr_cap : nullptr;
  uint8_t* xs_g = P.xscr ? reinterpret_cast<uint8_t*>(reinterpret_cast<XCand*>(P.xscr) + size_t(gridDim.x) * 2 *
                                                      P.xscr_cap) + size_t(blockIdx.x) * P.xscr_cap
                         : nullptr;
  uint32_t nbar = 0;
  load_slices(P, s_slc);
  __syncthreads();
  if (tid == 0) {
    mbar_init(&S->full[0]);
    mbar_init(&S->full[1]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (L > 1) {
      const int4 c = slice_of(P, s_slc, 1);
      fwd_issue(P, S, 1, c.x, c.y, c.z, c.w);
      for (int a = 1; a <= kSXAhead && a < L; ++a) {
        const int4 d = slice_of(P, s_slc, a);
        sx_prefetch_rec(P, d.z, d.w);
      }
    }
  }
  for (int s = gt; s < L; s += nthr) P.sl_cnt[s] = 0u;   // a full pass supersedes pending flags
  // startpoints: clock arrival distribution, mean and variance per rf
  for (int i = gt; i < P.num_src; i += nthr) {
    const float4 v = __ldg(P.src_ms + i);
    st_state(P.state + i, double(v.x), double(v.y), double(v.z) * double(v.z), double(v.w) * double(v.w), P.par);
  }
  uint32_t phase[2] = {0u, 0u};
  unsigned long long* ph = nullptr;
  for (int s = 1; s < L; ++s) {
    const int bf = s & 1;
    __syncthreads();   // level s - 1 is done with buffer bf ^ 1 and the candidate slots
#ifdef INSTA_SL_PHASES
    if (ph) ph[5] = gtimer();   // debug: the CTA finished level s - 1
#endif
    if (tid == 0 && s + 1 < L) {
      const int4 c = slice_of(P, s_slc, s + 1);
      fwd_issue(P, S, bf ^ 1, c.x, c.y, c.z, c.w);
      if (kSXPrefetch && s + kSXAhead < L) {
        const int4 d = slice_of(P, s_slc, s + kSXAhead);
        sx_prefetch_rec(P, d.z, d.w);
      }
    }
    if (!kFlow) grid_sync(P.bar, ++nbar, P.trace);   // levels < s are complete
#ifdef INSTA_SL_PHASES
    if (P.trace && tid == 0) {   // debug: per (level, CTA) timestamps
      ph = P.trace + 512 + size_t(L + 8) * 2 * gridDim.x + (size_t(s) * gridDim.x + blockIdx.x) * 8;
      ph[0] = gtimer();
    }
#endif
    const int4 sc = slice_of(P, s_slc, s);
    const int a = sc.x, b = sc.y, xa = sc.z, xb = sc.w;
    mbar_wait(&S->full[bf], phase[bf]);
    phase[bf] ^= 1u;
#ifdef INSTA_SL_PHASES
    if (ph) ph[2] = gtimer();
#endif
    if (b <= a) continue;
    const bool ok = S->ok[bf] != 0;
    const Window wp = window(a, b + 1, 4), wh = window(a, b, 4), wx = window(xa, xb, 4);
    // topology of the slice, indexed by head / entry id: staged, or global
    const int32_t* Pt = ok ? S->ptr[bf] + wp.off - a : P.hd_ptr;
    const int32_t* Pn = ok ? S->pin[bf] + wh.off - a : P.hd_pin;
    const int32_t* Wx = ok ? S->w[bf] + wx.off - xa : P.ext_w;
    const int32_t* Fx = ok ? S->f[bf] + wx.off - xa : P.ext_f;
    const bool fit = xb - xa <= kXCap;
    if (fit) sx_level<kLSE, kFlow>(P, a, b, xa, xb, Pt, Pn, Wx, Fx, xc_s - 2 * ptrdiff_t(xa), xs_s - ptrdiff_t(xa), ph);
    else sx_level<kLSE, kFlow>(P, a, b, xa, xb, Pt, Pn, Wx, Fx, xc_g - 2 * ptrdiff_t(xa), xs_g - ptrdiff_t(xa), ph);
  }
  grid_exit(P.bar);
}

// --------------------------------------------------------------------------
// One-cell what-if candidates (insta_eval_candidates; SURVEY §8(f) C5
// INSTA-Size "estimate the timing of each candidate"), all in ONE persistent
// launch.  Per candidate i (stamps 2i / 2i + 1 past the graph's epoch):
//   A  save the records of its arcs                          | barrier
//   B  write its records, stamp the heads evaluating them     | barrier
//   C  cone pass (levels flagged, one barrier per level)      | barrier
//   D  clear the level flags; recompute the flagged slack blocks' partials
//      (slack_common.cuh: the same per-block arithmetic as slack_kernel)  | barrier
//   E  CTA 0: the final slack reduction -> cand_out[i]; every CTA: write the
//      saved records back, stamp                              | barrier
//   F  cone pass again (reverts every record)                 | barrier
//   G  clear the level flags; recompute the flagged blocks again (base
//      partials, slack and rf* restored bit for bit); then A of i + 1.
// The flagged-block set is cleared in B of the next candidate (read in D, G).
// --------------------------------------------------------------------------
template <bool kLSE>
__device__ __forceinline__ void eval_apply(const SLParams& P, int i, bool revert, uint32_t stamp) {
  const int a0 = __ldg(P.cand_ptr + i), a1 = __ldg(P.cand_ptr + i + 1);
  for (int k = a0 + blockIdx.x * blockDim.x + threadIdx.x; k < a1; k += gridDim.x * blockDim.x) {
    const int id = __ldg(P.cand_arc + k);
    float4 r;
    if (revert) {
      r = P.cand_old[k];
    } else {
      const float2 m = __ldg(P.cand_m + k), sg = __ldg(P.cand_s + k);
      r = make_float4(m.x, m.y, sg.x, sg.y);
    }
    P.fin_ms[__ldg(P.arc_pos + id)] = r;
    const int x = __ldg(P.arc_xpos + id);   // the stage-folded schedule's copy of the record
    ((x & 1) ? P.ext_fms_w : P.ext_ms_w)[x >> 1] = r;
    const int h = __ldg(P.arc_head + id);
    P.dirty[h] = stamp;
    int lo = 0, hi = P.num_sl;   // its super-level is flagged
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (__ldg(P.sl_ptr + mid) <= h) lo = mid;
      else hi = mid;
    }
    atomicOr(P.sl_cnt + lo, 1u);
  }
}

__device__ __forceinline__ void eval_save(const SLParams& P, int i) {
  const int a0 = __ldg(P.cand_ptr + i), a1 = __ldg(P.cand_ptr + i + 1);
  for (int k = a0 + blockIdx.x * blockDim.x + threadIdx.x; k < a1; k += gridDim.x * blockDim.x)
    P.cand_old[k] = __ldcg(P.fin_ms + __ldg(P.arc_pos + __ldg(P.cand_arc + k)));
}

// flagged slack blocks of this CTA (b = blockIdx.x, blockIdx.x + grid, ...)
__device__ __forceinline__ void eval_slack_blocks(const SLParams& P, SlackRed& sr) {
  for (int b = blockIdx.x; b < P.slack_nb; b += gridDim.x) {
    if (!((__ldcg(P.ep_blk + (b >> 5)) >> (b & 31)) & 1u)) continue;
    slack_block(b, P.slack_nb, P.num_ep, P.ep_pin, P.ep_rat, P.state, double(P.n_sigma), P.slack, P.rf_star,
                P.partials, sr);
  }
}

template <bool kLSE>
__global__ void __launch_bounds__(kSLFwdThreads, 1) eval_kernel(SLParams P) {
  extern __shared__ __align__(128) unsigned char sl_smem[];
  __shared__ ConeSm cs;
  __shared__ SlackRed sr;
  int4* s_slc = reinterpret_cast<int4*>(sl_smem);
  int32_t* s_slp = reinterpret_cast<int32_t*>(s_slc + kSliceCap);
  const int tid = threadIdx.x, gt = blockIdx.x * blockDim.x + tid, nthr = gridDim.x * blockDim.x;
  const int L = P.num_sl, nw = (P.slack_nb + 31) / 32;
  load_slices(P, s_slc);
  for (int v = tid; v <= min(P.num_sl, kSliceCap); v += blockDim.x) s_slp[v] = __ldg(P.sl_ptr + v);
  uint32_t nbar = 0, nrec = 0;
  if (P.num_cand > 0) eval_save(P, 0);
  for (int i = 0; i < P.num_cand; ++i) {
    grid_sync(P.bar, ++nbar, P.trace);                                          // A done
    for (int w = gt; w < nw; w += nthr) P.ep_blk[w] = 0u;                      // read in D, G of i - 1
    for (int k = tid; k < 2 * kMarkWords; k += blockDim.x) cs.mark[k] = cs.pub[k] = 0u;
    if (P.elog && gt < 2) P.elog_n[gt] = 0u;                                    // read in E of i - 1
    eval_apply<kLSE>(P, i, false, P.stamp + 2 * i);
    grid_sync(P.bar, ++nbar, P.trace);                                          // B done
    cone_levels<kLSE>(P, P.stamp + 2 * i, cs, s_slc, s_slp, nbar, nrec);
    grid_sync(P.bar, ++nbar, P.trace);                                          // C done
    for (int s = gt; s < L; s += nthr) P.sl_cnt[s] = 0u;
    eval_slack_blocks(P, sr);
    grid_sync(P.bar, ++nbar, P.trace);                                          // D done
    if (blockIdx.x == 0) slack_final(P.slack_nb, P.partials, P.cand_out + 3 * size_t(i), sr);
    for (int k = tid; k < 2 * kMarkWords; k += blockDim.x) cs.mark[k] = cs.pub[k] = 0u;
    eval_apply<kLSE>(P, i, true, P.stamp + 2 * i + 1);
    const uint32_t n0 = P.elog ? __ldcg(P.elog_n) : 0u, n1 = P.elog ? __ldcg(P.elog_n + 1) : 0u;
    if (P.elog && n0 <= uint32_t(P.elog_cap) && n1 <= uint32_t(P.elog_cap)) {
      // undo log: every record and arg-max word the cone pass overwrote, written back (each head /
      // entry appears once: a cone pass recomputes a head at most once)
      for (uint32_t k = gt; k < n0; k += nthr) {
        const EvLog e = P.elog[k];
        asm volatile("st.relaxed.gpu.global.v4.b64 [%0], {%1, %2, %3, %4};" ::"l"(P.state + e.pin), "l"(e.rec.a),
                     "l"(e.rec.b), "l"(e.rec.c), "l"(e.rec.d)
                     : "memory");
        P.hwin[e.h] = e.win;
      }
      for (uint32_t k = gt; k < n1; k += nthr) {
        const int2 f = P.flog[k];
        P.fwin[f.x] = f.y;
      }
      grid_sync(P.bar, ++nbar, P.trace);                                        // E, F done
    } else {   // no log (LSE) or it overflowed: the cone pass again reverts every record
      grid_sync(P.bar, ++nbar, P.trace);                                        // E done
      cone_levels<kLSE>(P, P.stamp + 2 * i + 1, cs, s_slc, s_slp, nbar, nrec);
      grid_sync(P.bar, ++nbar, P.trace);                                        // F done
    }
    for (int s = gt; s < L; s += nthr) P.sl_cnt[s] = 0u;
    eval_slack_blocks(P, sr);
    if (i + 1 < P.num_cand) eval_save(P, i + 1);
  }
  grid_sync(P.bar, ++nbar, P.trace);
  for (int w = gt; w < nw; w += nthr) P.ep_blk[w] = 0u;
  grid_exit(P.bar);
}

// --------------------------------------------------------------------------
// Backward
// --------------------------------------------------------------------------
constexpr int kSLHeavyTab = 256;
struct SLHeavyTab {
  int32_t key[kSLHeavyTab];
  unsigned long long acc[kSLHeavyTab][2];
};

__device__ __forceinline__ void red_u64(unsigned long long* a, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(a), "l"(v));
}

__device__ __forceinline__ void push_adj(const SLParams& P, SLHeavyTab* tab, int sh, bool heavy, float gx, float gy) {
  if (gx == 0.f && gy == 0.f) return;
  const unsigned long long vx = (unsigned long long)__double2ll_rn(double(gx) * kAccScale);
  const unsigned long long vy = (unsigned long long)__double2ll_rn(double(gy) * kAccScale);
  if (heavy) {   // a driver with > kHeavyFanout sinks: combine in shared memory first
    int hh = int((uint32_t(sh) * 2654435761u) >> 24) & (kSLHeavyTab - 1);
    for (int probe = 0; probe < 8; ++probe, hh = (hh + 1) & (kSLHeavyTab - 1)) {
      const int prev = atomicCAS(&tab->key[hh], -1, sh);
      if (prev == -1 || prev == sh) {
        atomicAdd(&tab->acc[hh][0], vx);
        atomicAdd(&tab->acc[hh][1], vy);
        return;
      }
    }
  }
  unsigned long long* a = reinterpret_cast<unsigned long long*>(P.acc) + 2 * size_t(sh);
  red_u64(a, vx);
  red_u64(a + 1, vy);
}

__device__ __forceinline__ void heavy_flush(const SLParams& P, SLHeavyTab* tab) {
  for (int k = threadIdx.x; k < kSLHeavyTab; k += blockDim.x) {
    const int sh = tab->key[k];
    if (sh >= 0) {
      unsigned long long* a = reinterpret_cast<unsigned long long*>(P.acc) + 2 * size_t(sh);
      red_u64(a, tab->acc[k][0]);
      red_u64(a + 1, tab->acc[k][1]);
      tab->key[k] = -1;
      tab->acc[k][0] = 0ull;
      tab->acc[k][1] = 0ull;
    }
  }
}

// Eq 6 sink side of one arc: weights w[rf][s] (hard: selection bits, bit
// 2 rf + s; LSE: w4), dL/d(arc mean) written when nonzero (the prologue zero
// fills), returns the adjoint to the source's {R, F}.
template <bool kLSE>
__device__ __forceinline__ float2 sl_sink(const SLParams& P, float2 ab, int sel, float4 w4, int32_t arcid) {
  const float abr[2] = {ab.x, ab.y};
  float w[2][2];
  if (kLSE) {
    w[0][0] = w4.x;
    w[0][1] = w4.y;
    w[1][0] = w4.z;
    w[1][1] = w4.w;
  } else {
#pragma unroll
    for (int rf = 0; rf < 2; ++rf) {
      w[rf][0] = ((sel >> (2 * rf)) & 1) ? 1.f : 0.f;
      w[rf][1] = ((sel >> (2 * rf + 1)) & 1) ? 1.f : 0.f;
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
  if (gm[0] != 0.f || gm[1] != 0.f) reinterpret_cast<float2*>(P.d_mean)[arcid] = make_float2(gm[0], gm[1]);
  return make_float2(gs[0], gs[1]);
}

__device__ __forceinline__ int sel_of(int32_t win, int k) {
  int sel = 0;
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    const int wv = (win >> (16 * rf)) & 0xffff;
    if ((wv & 0x7fff) == k) sel |= 1 << (2 * rf + (wv >> 15));
  }
  return sel;
}

// selection / weights of a unate folding arc e' (its single candidate per rf
// is s0 = src_tr(rf, u, 0): POS {R<-R, F<-F}, NEG {R<-F, F<-R})
__device__ __forceinline__ int unate_sel(int u) { return u == 1 ? (0x2 | 0x4) : (0x1 | 0x8); }
__device__ __forceinline__ float4 unate_w(int u) {
  return u == 1 ? make_float4(0.f, 1.f, 1.f, 0.f) : make_float4(1.f, 0.f, 0.f, 1.f);
}

// backward stage: head rows, seeds, arg-max words; entry topology and weights
constexpr int kBRowCap = 1024, kBEntCap = 2048;
struct BStage {
  int32_t ptr[kBRowCap + 8];
  float2 seed[kBRowCap + 8];
  int32_t win[kBRowCap + 8];
  int32_t arc[kBEntCap + 8];
  int32_t farc[kBEntCap + 8];
  int32_t sh[kBEntCap + 8];
  int32_t bw[kBEntCap + 8];
  int32_t f[kBEntCap + 8];
  float4 w4[kBEntCap];
};
struct BStageSet {
  BStage st[2];
  uint64_t full[2];
  int32_t ok[2];
};
constexpr size_t kBSlcOff = (sizeof(BStageSet) + 15) & ~size_t(15);
constexpr size_t kBStageBytes = kBSlcOff + sizeof(int4) * kSliceCap;

template <bool kLSE>
__device__ __forceinline__ void bwd_issue(const SLParams& P, BStageSet* S, int bf, int a, int b, int xa, int xb) {
  const bool fits = b > a && b - a <= kBRowCap && xb - xa <= kBEntCap;
  S->ok[bf] = fits ? 1 : 0;
  if (!fits) {
    mbar_arrive(&S->full[bf]);
    return;
  }
  const Window wp = window(a, b + 1, 4), wh = window(a, b, 4), ws = window(a, b, 8), wx = window(xa, xb, 4);
  const uint32_t bw4 = kLSE ? uint32_t(xb - xa) * 16u : 0u;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mbar_expect_tx(&S->full[bf], wp.bytes + ws.bytes + (kLSE ? 0u : wh.bytes) + 5 * wx.bytes + bw4);
  BStage& T = S->st[bf];
  bulk_g2s(T.ptr, P.hd_ptr + wp.start, wp.bytes, &S->full[bf]);
  bulk_g2s(T.seed, P.hseed + ws.start, ws.bytes, &S->full[bf]);
  if (!kLSE) bulk_g2s(T.win, P.hwin + wh.start, wh.bytes, &S->full[bf]);
  if (wx.bytes) {
    bulk_g2s(T.arc, P.ext_arc + wx.start, wx.bytes, &S->full[bf]);
    bulk_g2s(T.farc, P.ext_farc + wx.start, wx.bytes, &S->full[bf]);
    bulk_g2s(T.sh, P.ext_sh + wx.start, wx.bytes, &S->full[bf]);
    bulk_g2s(T.bw, P.ext_bw + wx.start, wx.bytes, &S->full[bf]);
    bulk_g2s(T.f, P.ext_f + wx.start, wx.bytes, &S->full[bf]);
  }
  if (bw4) bulk_g2s(T.w4, P.ew + xa, bw4, &S->full[bf]);
}

// Backward of one head: its adjoint (seed + consumers' shares, read and
// cleared), then the Eq 6 sink side of every entry (through the folded pin
// when there is one) and the share pushed to the entry's source head.
// T: the staged slice (entry words at xr + k, weights at xw + k) or nullptr (global).
template <bool kLSE>
__device__ __forceinline__ void sl_bwd_head(const SLParams& P, SLHeavyTab* tab, int h, int x0, int nf, float2 sd,
                                            int32_t win, const BStage* T, int xr, int xw) {
  unsigned long long ax, ay;
  ld2_u64(P.acc + 2 * size_t(h), ax, ay);
  if (ax | ay) asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %1};" ::"l"(P.acc + 2 * size_t(h)), "l"(0ull));
  const float2 ab = make_float2(sd.x + float(double((long long)ax) * kAccInv),
                                sd.y + float(double((long long)ay) * kAccInv));
  if (P.acc_b) {   // snapshot for insta_backward_update
    asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(P.acc_b + 2 * size_t(h)), "l"(ax), "l"(ay) : "memory");
    P.hab_b[h] = ab;
  }
  // nothing flows through this head: its arcs keep the zero prefill (scattered zero stores in
  // caller arc order cost 2.5x the whole backward on B200: measured, profiles/r02_summary.md)
  if (ab.x == 0.f && ab.y == 0.f) return;
  for (int k = 0; k < nf; ++k) {
    const int x = x0 + k;
    int32_t arc, farc, sh, bw, f;
    float4 w4 = make_float4(0.f, 0.f, 0.f, 0.f);
    if (T) {
      arc = T->arc[xr + k];
      farc = T->farc[xr + k];
      sh = T->sh[xr + k];
      bw = T->bw[xr + k];
      f = T->f[xr + k];
      if (kLSE) w4 = T->w4[xw + k];
    } else {
      arc = __ldg(P.ext_arc + x);
      farc = __ldg(P.ext_farc + x);
      sh = __ldg(P.ext_sh + x);
      bw = __ldg(P.ext_bw + x);
      f = __ldg(P.ext_f + x);
      if (kLSE) w4 = __ldcg(P.ew + x);
    }
    float2 gs = sl_sink<kLSE>(P, ab, kLSE ? 0 : sel_of(win, k), w4, arc);
    if (farc >= 0) {   // through the folded pin p: its adjoint is gs, then the arc e' = (j -> p)
      const int u2 = int(uint32_t(f) >> kUnateShift);
      int fsel = 0;
      float4 fw = make_float4(0.f, 0.f, 0.f, 0.f);
      if (u2 != 2) {
        if (kLSE) fw = unate_w(u2);
        else fsel = unate_sel(u2);
      } else if (kLSE) {
        fw = __ldcg(P.efw + x);
      } else {
        fsel = sel_of(__ldcg(P.fwin + x), 0);
      }
      gs = sl_sink<kLSE>(P, gs, fsel, fw, farc);
    }
    push_adj(P, tab, sh, (bw >> kHeavyBit) & 1, gs.x, gs.y);
  }
}

template <bool kLSE>
__global__ void __launch_bounds__(kSLBwdThreads, 1) bwdl_kernel(SLParams P) {
  extern __shared__ __align__(128) unsigned char sl_smem[];
  BStageSet* S = reinterpret_cast<BStageSet*>(sl_smem);
  __shared__ SLHeavyTab tab;
  const int tid = threadIdx.x;
  for (int k = tid; k < kSLHeavyTab; k += blockDim.x) {
    tab.key[k] = -1;
    tab.acc[k][0] = 0ull;
    tab.acc[k][1] = 0ull;
  }
  const int L = P.num_sl;
  uint32_t nbar = 0;
  if (P.trace && blockIdx.x == 0 && tid == 0) P.trace[0] = gtimer();
  int4* s_slc = reinterpret_cast<int4*>(sl_smem + kBSlcOff);
  load_slices(P, s_slc);
  __syncthreads();
  if (tid == 0) {
    mbar_init(&S->full[0]);
    mbar_init(&S->full[1]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (L > 1) {
      const int4 c = slice_of(P, s_slc, L - 1);
      bwd_issue<kLSE>(P, S, (L - 1) & 1, c.x, c.y, c.z, c.w);
    }
  }
  uint32_t phase[2] = {0u, 0u};
  for (int s = L - 1; s >= 1; --s) {
    const int bf = s & 1;
    __syncthreads();   // every thread is done with buffer bf ^ 1 (level s + 1)
    if (tid == 0 && s - 1 >= 1) {   // stage level s - 1 while level s runs
      const int4 c = slice_of(P, s_slc, s - 1);
      bwd_issue<kLSE>(P, S, bf ^ 1, c.x, c.y, c.z, c.w);
    }
    if (s < L - 1) grid_sync(P.bar, ++nbar, P.trace);   // levels > s are complete
    mbar_wait(&S->full[bf], phase[bf]);
    phase[bf] ^= 1u;
    const int4 sc = slice_of(P, s_slc, s);
    const int a = sc.x, b = sc.y;
    if (b > a) {
      const BStage& T = S->st[bf];
      if (S->ok[bf]) {
        const Window wp = window(a, b + 1, 4), wh = window(a, b, 4), ws = window(a, b, 8);
        const int xa = sc.z;
        const Window wx = window(xa, sc.w, 4);
        for (int h = a + tid; h < b; h += blockDim.x) {
          const int r = h - a;
          const int x0 = T.ptr[wp.off + r], nf = T.ptr[wp.off + r + 1] - x0;
          const int32_t win = kLSE ? 0 : T.win[wh.off + r];
          sl_bwd_head<kLSE>(P, &tab, h, x0, nf, T.seed[ws.off + r], win, &T, wx.off + x0 - xa, x0 - xa);
        }
      } else {
        for (int h = a + tid; h < b; h += blockDim.x) {
          const int x0 = __ldg(P.hd_ptr + h), nf = __ldg(P.hd_ptr + h + 1) - x0;
          sl_bwd_head<kLSE>(P, &tab, h, x0, nf, P.hseed[h], kLSE ? 0 : __ldcg(P.hwin + h), nullptr, 0, 0);
        }
      }
    }
    __syncthreads();
    heavy_flush(P, &tab);
  }
  // level 0 (startpoints, hd_pin[h] = h): dL/d(source mean)
  if (L > 1) grid_sync(P.bar, ++nbar, P.trace);
  for (int h = blockIdx.x * blockDim.x + tid; h < P.num_src; h += gridDim.x * blockDim.x) {
    unsigned long long ax, ay;
    ld2_u64(P.acc + 2 * size_t(h), ax, ay);
    if (ax | ay) asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %1};" ::"l"(P.acc + 2 * size_t(h)), "l"(0ull));
    const float2 sd = P.hseed[h];
    if (P.acc_b) {
      asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(P.acc_b + 2 * size_t(h)), "l"(ax), "l"(ay) : "memory");
      P.hab_b[h] = make_float2(sd.x + float(double((long long)ax) * kAccInv), sd.y + float(double((long long)ay) * kAccInv));
    }
    if (P.d_src)
      reinterpret_cast<float2*>(P.d_src)[__ldg(P.order + h)] =
          make_float2(sd.x + float(double((long long)ax) * kAccInv), sd.y + float(double((long long)ay) * kAccInv));
  }
  grid_exit(P.bar);
}

// --------------------------------------------------------------------------
// Incremental backward (insta_backward_update; SURVEY §8(f) NEXT 3
// INSTA-Size, P:L229 incremental evaluation).
//
// The sweep backward accumulates every head's adjoint as an integer sum of
// fixed-point shares (push_adj), so a later backward can be reached exactly by
// deltas: a snapshot backward keeps, per head, its accumulated sum (acc_b), its
// adjoint (hab_b), seed and arg-max word, and per entry the folded arg-max /
// Eq 6 weights.  After cone passes (which stamp the heads they recompute), the
// update (1) recomputes the endpoint seeds, (2) marks every touched head whose
// seed, arg-max or weights differ from the snapshot, then (3) walks the flagged
// super-levels in reverse: a marked head adds the deltas pushed to it to its
// sum, forms its adjoint exactly as the full backward does, rewrites dL/d(mean)
// of its arcs, and pushes fix(new share) - fix(old share) to each source --
// marking the source when that difference is nonzero.  Integer addition is
// exact and order-free, so every sum, adjoint and gradient equals the full
// backward's bit for bit; the work is the reverse cone of the change, cut off
// where the shares stop changing.
// --------------------------------------------------------------------------
__device__ __forceinline__ long long fixp(float v) { return __double2ll_rn(double(v) * kAccScale); }

// sl_sink with the store of dL/d(mean) optional and unconditional (zeros included)
template <bool kLSE>
__device__ __forceinline__ float2 bi_sink(const SLParams& P, float2 ab, int sel, float4 w4, int32_t arcid, bool store) {
  const float abr[2] = {ab.x, ab.y};
  float w[2][2];
  if (kLSE) {
    w[0][0] = w4.x;
    w[0][1] = w4.y;
    w[1][0] = w4.z;
    w[1][1] = w4.w;
  } else {
#pragma unroll
    for (int rf = 0; rf < 2; ++rf) {
      w[rf][0] = ((sel >> (2 * rf)) & 1) ? 1.f : 0.f;
      w[rf][1] = ((sel >> (2 * rf + 1)) & 1) ? 1.f : 0.f;
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
  // the full backward stores a nonzero pair as is and leaves the zero prefill otherwise
  if (store)
    reinterpret_cast<float2*>(P.d_mean)[arcid] =
        (gm[0] != 0.f || gm[1] != 0.f) ? make_float2(gm[0], gm[1]) : make_float2(0.f, 0.f);
  return make_float2(gs[0], gs[1]);
}

__device__ __forceinline__ void bi_mark(const SLParams& P, const int32_t* s_slp, int h) {
  P.bdirty[h] = P.bstamp;
  atomicOr(P.bl_cnt + sl_of(P, s_slp, h), 1u);
}

// (2) heads recomputed since the snapshot whose seed, arg-max or weights differ
template <bool kLSE>
__global__ void __launch_bounds__(256) bdiff_kernel(SLParams P) {
  __shared__ int32_t s_slp[kSliceCap + 4];
  for (int v = threadIdx.x; v <= min(P.num_sl, kSliceCap); v += blockDim.x) s_slp[v] = __ldg(P.sl_ptr + v);
  __syncthreads();
  for (int h = blockIdx.x * blockDim.x + threadIdx.x; h < P.num_heads; h += gridDim.x * blockDim.x) {
    if (__ldcg(P.btouch + h) != P.bepoch) continue;
    const float2 a = P.hseed[h], b = P.hseed_b[h];
    bool chg = __float_as_uint(a.x) != __float_as_uint(b.x) || __float_as_uint(a.y) != __float_as_uint(b.y);
    if (!kLSE) chg |= __ldcg(P.hwin + h) != P.hwin_b[h];
    const int x0 = __ldg(P.hd_ptr + h), x1 = __ldg(P.hd_ptr + h + 1);
    for (int x = x0; x < x1 && !chg; ++x) {
      if (kLSE) {
        const float4 u = __ldcg(P.ew + x), v = P.ew_b[x];
        chg |= __float_as_uint(u.x) != __float_as_uint(v.x) || __float_as_uint(u.y) != __float_as_uint(v.y) ||
               __float_as_uint(u.z) != __float_as_uint(v.z) || __float_as_uint(u.w) != __float_as_uint(v.w);
      }
      if (__ldg(P.ext_farc + x) >= 0 && (uint32_t(__ldg(P.ext_f + x)) >> kUnateShift) == 2u) {   // non-unate folded arc
        if (kLSE) {
          const float4 u = __ldcg(P.efw + x), v = P.efw_b[x];
          chg |= __float_as_uint(u.x) != __float_as_uint(v.x) || __float_as_uint(u.y) != __float_as_uint(v.y) ||
                 __float_as_uint(u.z) != __float_as_uint(v.z) || __float_as_uint(u.w) != __float_as_uint(v.w);
        } else {
          chg |= __ldcg(P.fwin + x) != P.fwin_b[x];
        }
      }
    }
    if (chg) bi_mark(P, s_slp, h);
  }
}

// (3) one marked head: its adjoint from the snapshot sum plus the pushed deltas,
// its arcs' gradients, and the share deltas to its sources; the snapshot follows
template <bool kLSE>
__device__ __forceinline__ int bi_head(const SLParams& P, const int32_t* s_slp, int h) {
  unsigned long long dx, dy;
  ld2_u64(P.acc + 2 * size_t(h), dx, dy);
  if (dx | dy) asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %1};" ::"l"(P.acc + 2 * size_t(h)), "l"(0ull));
  const long long tx = P.acc_b[2 * size_t(h)] + (long long)dx, ty = P.acc_b[2 * size_t(h) + 1] + (long long)dy;
  P.acc_b[2 * size_t(h)] = tx;
  P.acc_b[2 * size_t(h) + 1] = ty;
  const float2 sd = P.hseed[h];
  const float2 ab = make_float2(sd.x + float(double(tx) * kAccInv), sd.y + float(double(ty) * kAccInv));
  const float2 ao = P.hab_b[h];
  P.hab_b[h] = ab;
  P.hseed_b[h] = sd;
  if (h < P.num_src) return 0;   // a startpoint: no arcs
  int32_t wn = 0, wo = 0;
  if (!kLSE) {
    wn = __ldcg(P.hwin + h);
    wo = P.hwin_b[h];
    P.hwin_b[h] = wn;
  }
  const int x0 = __ldg(P.hd_ptr + h), nf = __ldg(P.hd_ptr + h + 1) - x0;
  for (int k = 0; k < nf; ++k) {
    const int x = x0 + k;
    const int32_t arc = __ldg(P.ext_arc + x), farc = __ldg(P.ext_farc + x), sh = __ldg(P.ext_sh + x);
    float4 w4n = make_float4(0.f, 0.f, 0.f, 0.f), w4o = w4n;
    if (kLSE) {
      w4n = __ldcg(P.ew + x);
      w4o = P.ew_b[x];
      P.ew_b[x] = w4n;
    }
    float2 gn = bi_sink<kLSE>(P, ab, kLSE ? 0 : sel_of(wn, k), w4n, arc, true);
    float2 go = bi_sink<kLSE>(P, ao, kLSE ? 0 : sel_of(wo, k), w4o, arc, false);
    if (farc >= 0) {   // through the folded pin (as sl_bwd_head)
      const int u2 = int(uint32_t(__ldg(P.ext_f + x)) >> kUnateShift);
      int fsn = 0, fso = 0;
      float4 fwn = make_float4(0.f, 0.f, 0.f, 0.f), fwo = fwn;
      if (u2 != 2) {
        if (kLSE) fwn = fwo = unate_w(u2);
        else fsn = fso = unate_sel(u2);
      } else if (kLSE) {
        fwn = __ldcg(P.efw + x);
        fwo = P.efw_b[x];
        P.efw_b[x] = fwn;
      } else {
        const int32_t a = __ldcg(P.fwin + x), b = P.fwin_b[x];
        P.fwin_b[x] = a;
        fsn = sel_of(a, 0);
        fso = sel_of(b, 0);
      }
      gn = bi_sink<kLSE>(P, gn, fsn, fwn, farc, true);
      go = bi_sink<kLSE>(P, go, fso, fwo, farc, false);
    }
    const long long ddx = fixp(gn.x) - fixp(go.x), ddy = fixp(gn.y) - fixp(go.y);
    if (ddx | ddy) {
      unsigned long long* a = reinterpret_cast<unsigned long long*>(P.acc) + 2 * size_t(sh);
      red_u64(a, (unsigned long long)ddx);
      red_u64(a + 1, (unsigned long long)ddy);
      if (__ldcg(P.bdirty + sh) != P.bstamp) bi_mark(P, s_slp, sh);
    }
  }
  return 1;
}

template <bool kLSE>
__global__ void __launch_bounds__(kSLBwdThreads, 1) bwdi_kernel(SLParams P) {
  __shared__ int4 s_slc[kSliceCap];
  __shared__ int32_t s_slp[kSliceCap + 4];
  __shared__ int32_t s_next;
  const int tid = threadIdx.x, L = P.num_sl;
  uint32_t nbar = 0, nrun = 0;
  load_slices(P, s_slc);
  for (int v = tid; v <= min(P.num_sl, kSliceCap); v += blockDim.x) s_slp[v] = __ldg(P.sl_ptr + v);
  __syncthreads();
  int s = L;   // levels >= s are done
  for (;;) {
    // next flagged level below s: every flag there is final (set by levels >= s, before the last barrier)
    if (tid < 32) {
      int nx = -1;
      for (int top = s - 1; top >= 0; top -= 32) {
        const int lv = top - tid;
        const uint32_t f = lv >= 0 ? __ldcg(P.bl_cnt + lv) : 0u;
        const uint32_t hit = __ballot_sync(0xffffffffu, f != 0u);
        if (hit) {
          nx = top - (__ffs(hit) - 1);
          break;
        }
      }
      if (tid == 0) s_next = nx;
    }
    __syncthreads();
    s = s_next;
    __syncthreads();
    if (s < 0) break;
    const int4 sc = slice_of(P, s_slc, s);
    for (int h = sc.x + tid; h < sc.y; h += blockDim.x)
      if (__ldcg(P.bdirty + h) == P.bstamp) nrun += uint32_t(bi_head<kLSE>(P, s_slp, h));
    grid_sync(P.bar, ++nbar, P.trace);   // level s is complete: its pushes and marks are visible
  }
  for (int v = blockIdx.x * blockDim.x + tid; v < L; v += gridDim.x * blockDim.x) P.bl_cnt[v] = 0u;
  const uint32_t n = __reduce_add_sync(0xffffffffu, nrun);
  if ((tid & 31) == 0 && n) atomicAdd(P.counters + 2, (unsigned long long)n);
  grid_exit(P.bar);
}

// Folded pins' records, arg-max and Eq 6 weights from their sources' records
// (a sweep forward does not store them): one thread per entry.
template <bool kLSE>
__global__ void __launch_bounds__(256) fold_fill_kernel(SLParams P, int64_t num_ext) {
  const int64_t x = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (x >= num_ext) return;
  const int32_t w = __ldg(P.ext_w + x);
  if (!((w >> kFoldBit) & 1)) return;
  SLParams Q = P;
  Q.store_fold = 1;
  (void)sl_fold<kLSE>(Q, __ldg(P.ext_f + x), P.ext_fms[x], int(x), ld_raw(P.state + (w & kSrcMask)));
}

// --------------------------------------------------------------------------
// Launchers
// --------------------------------------------------------------------------
static SLParams sl_params(DevGraph& g) {
  SLParams P{};
  P.num_sl = g.num_slevels;
  P.num_src = g.num_src;
  P.num_heads = g.num_heads;
  P.sl_ptr = g.sl_ptr;
  P.slice = g.sl_slice;
  P.hd_ptr = g.hd_ptr;
  P.hd_pin = g.hd_pin;
  P.hd_q0 = g.hd_q0;
  P.ext_w = g.ext_w;
  P.ext_ms = g.ext_ms;
  P.ext_f = g.ext_f;
  P.ext_fms = g.ext_fms;
  P.ext_fq = g.ext_fq;
  P.src_ms = g.src_ms;
  P.state = g.state;
  P.win = g.win;
  P.wts = g.wts;
  P.hwin = g.hwin;
  P.ew = g.ew;
  P.fwin = g.fwin;
  P.efw = g.efw;
  P.bar = g.sl_bar;
  P.dirty = g.dirty_h;
  P.hd_csl = g.hd_csl;
  P.hfo_ptr = g.hfo_ptr;
  P.hfo = g.hfo;
  P.hfo_sl = g.hfo_sl;
  P.hd_hsrc = g.hd_hsrc;
  P.chg = g.chg;
  P.sl_cnt = g.sl_cnt;
  P.counters = g.counters;
  P.ext_arc = g.ext_arc;
  P.ext_farc = g.ext_farc;
  P.ext_sh = g.ext_sh;
  P.ext_bw = g.ext_bw;
  P.order = g.order;
  P.hseed = g.hseed;
  P.acc = g.acc_h;
  P.store_fold = 0;
  P.hd_eop = g.hd_eop;
  P.ep_blk = nullptr;
  P.slack_nb = slack_blocks(g.num_ep, g.sl_grid > 0 ? g.sl_grid : 148);
  P.num_ep = g.num_ep;
  P.ep_pin = g.ep_pin;
  P.ep_rat = g.ep_rat;
  P.slack = g.slack;
  P.rf_star = g.rf_star;
  P.partials = g.partials;
  P.arc_pos = g.arc_pos;
  P.arc_xpos = g.arc_xpos;
  P.arc_head = g.arc_head;
  P.fin_ms = g.fin_ms;
  P.ext_ms_w = g.ext_ms;
  P.ext_fms_w = g.ext_fms;
  P.btouch = g.btouch;   // cone passes stamp the heads they recompute (incremental backward)
  P.bepoch = g.bepoch;
  return P;
}

template <class K>
static cudaError_t sl_smem_attr(K kernel, size_t bytes) {
  return cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bytes));
}

constexpr size_t kEvalSmem = sizeof(int4) * kSliceCap + sizeof(int32_t) * (kSliceCap + 4);

int query_sl_grid(int device, int* grid_f, int* grid_b) {
  int sms = 0;
  cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  if (e == cudaSuccess) e = sl_smem_attr(fwdl_kernel<false, 0>, kFStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdl_kernel<true, 0>, kFStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdl_kernel<false, 1>, kFStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdl_kernel<true, 1>, kFStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdl_kernel<false, 2>, kFStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdl_kernel<true, 2>, kFStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdx_kernel<false, false>, kXStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdx_kernel<true, false>, kXStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdx_kernel<false, true>, kXStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(fwdx_kernel<true, true>, kXStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(eval_kernel<false>, kEvalSmem);
  if (e == cudaSuccess) e = sl_smem_attr(eval_kernel<true>, kEvalSmem);
  if (e == cudaSuccess) e = sl_smem_attr(bwdl_kernel<false>, kBStageBytes);
  if (e == cudaSuccess) e = sl_smem_attr(bwdl_kernel<true>, kBStageBytes);
  if (e != cudaSuccess) return int(e);
  int occ = 1 << 30, b = 0;
  const void* kf[] = {(const void*)fwdl_kernel<false, 0>, (const void*)fwdl_kernel<true, 0>,
                      (const void*)fwdl_kernel<false, 1>, (const void*)fwdl_kernel<true, 1>,
                      (const void*)fwdl_kernel<false, 2>, (const void*)fwdl_kernel<true, 2>};
  const size_t sf[] = {kFStageBytes, kFStageBytes, kFStageBytes, kFStageBytes, kFStageBytes, kFStageBytes};
  for (int i = 0; i < 6; ++i) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kf[i], kSLFwdThreads, sf[i]);
    if (e != cudaSuccess) return int(e);
    occ = std::min(occ, b);
  }
  const void* kx[] = {(const void*)fwdx_kernel<false, false>, (const void*)fwdx_kernel<true, false>,
                      (const void*)fwdx_kernel<false, true>, (const void*)fwdx_kernel<true, true>};
  for (int i = 0; i < 4; ++i) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kx[i], sx_threads(i & 1), kXStageBytes);
    if (e != cudaSuccess) return int(e);
    occ = std::min(occ, b);
  }
  if (occ <= 0) return int(cudaErrorLaunchOutOfResources);
  *grid_f = sms;   // one CTA per SM (the stage and the barrier arrival are per CTA)
  occ = 1 << 30;
  const void* kb[] = {(const void*)bwdl_kernel<false>, (const void*)bwdl_kernel<true>};
  for (int i = 0; i < 2; ++i) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kb[i], kSLBwdThreads, kBStageBytes);
    if (e != cudaSuccess) return int(e);
    occ = std::min(occ, b);
  }
  if (occ <= 0) return int(cudaErrorLaunchOutOfResources);
  *grid_b = sms;
  return 0;
}

// INSTA_SL_TRACE=<dir>: CTA 0's globaltimer at the start and at every barrier
// exit, and every CTA's arrival, written to <dir>/sl_<name>.bin (uint64; synchronizes)
static int launch_coop(const void* fn, int grid, int threads, size_t smem, SLParams& P, cudaStream_t st,
                       const char* name) {
  const char* dir = getenv("INSTA_SL_TRACE");
  const size_t nt = 512 + size_t(P.num_sl + 8) * 10 * size_t(grid);
  P.trace = nullptr;
  if (dir) {
    cudaMalloc(&P.trace, nt * 8);
    cudaMemsetAsync(P.trace, 0, nt * 8, st);
  }
  void* args[] = {&P};
  int err = int(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(threads), args, smem, st));
  if (dir && P.trace) {
    std::vector<unsigned long long> h(nt);
    cudaMemcpyAsync(h.data(), P.trace, nt * 8, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
    cudaFree(P.trace);
    std::string path = std::string(dir) + "/sl_" + name + ".bin";
    FILE* f = fopen(path.c_str(), "wb");
    if (f) {
      fwrite(h.data(), 8, nt, f);
      fclose(f);
    }
    P.trace = nullptr;
  }
  return err;
}

int launch_forward_sl(DevGraph& g, float n_sigma, float tau, void* stream, bool flow) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (g.n == 0) return 0;
  SLParams P = sl_params(g);
  P.n_sigma = n_sigma;
  P.tau = tau;
  P.inv_tau = tau > 0.f ? 1.0 / double(tau) : 0.0;
  P.par = (++g.pass_fwd) & 1u;
  ++g.inc_epoch;   // a full pass supersedes pending incremental marks
  const bool lse = tau > 0.f;
  if (g.sl_max_x > kXCap && !g.xscr) {   // candidate buffers of slices beyond shared memory
    const cudaError_t e =
        cudaMalloc(&g.xscr, size_t(g.sl_grid) * size_t(g.sl_max_x) * (2 * sizeof(XCand) + 1));
    if (e != cudaSuccess) return int(e);
  }
  P.xscr = g.sl_max_x > kXCap ? g.xscr : nullptr;
  P.xscr_cap = g.sl_max_x;
  // flow: no grid barrier (parity dataflow); needs uniform record parity (no cone pass since the last full pass)
  const void* fn = flow ? (lse ? (const void*)fwdx_kernel<true, true> : (const void*)fwdx_kernel<false, true>)
                        : (lse ? (const void*)fwdx_kernel<true, false> : (const void*)fwdx_kernel<false, false>);
  const int err = launch_coop(fn, g.sl_grid, sx_threads(lse), kXStageBytes, P, st, lse ? "fwd_lse" : "fwd");
  if (!err) g.parity_mixed = false;
  g.folded_valid = false;
  return err;
}

int launch_forward_cone(DevGraph& g, float n_sigma, float tau, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaMemsetAsync(g.counters, 0, sizeof(unsigned long long) * 2, st);
  if (e != cudaSuccess) return int(e);
  if (g.n == 0) return 0;
  SLParams P = sl_params(g);
  P.n_sigma = n_sigma;
  P.tau = tau;
  P.inv_tau = tau > 0.f ? 1.0 / double(tau) : 0.0;
  // the cone pass is ordered by its barriers, not by parity: it rewrites the
  // changed records with the CURRENT parity, so the records stay uniform and the
  // next dataflow pass (new parity) can wait on them
  P.par = g.pass_fwd & 1u;
  P.stamp = ++g.inc_epoch;
  const bool lse = tau > 0.f;
  // large update batches: stage every level's topology (latency off the chain);
  // small ones: read only the dirty heads' topology
  const bool staged = g.pending_updates * 1000 > g.e;
  const void* fn = staged ? (lse ? (const void*)fwdl_kernel<true, 1> : (const void*)fwdl_kernel<false, 1>)
                          : (lse ? (const void*)fwdl_kernel<true, 2> : (const void*)fwdl_kernel<false, 2>);
  if (g.slack_valid) P.ep_blk = g.ep_blk;   // insta_forward follows with the slack of the flagged blocks only
  const int err = launch_coop(fn, g.sl_grid, kSLFwdThreads, kFStageBytes, P, st, "cone");
  g.folded_valid = false;
  return err;
}

// All candidates in one persistent launch (eval_kernel).  cand_ptr: host; the
// arc arrays on the device.  Stamps past the graph's epoch, 2 per candidate.
int launch_eval_candidates(DevGraph& g, int num, const int32_t* cand_ptr, const int32_t* arc_ids, const float* mean,
                           const float* sigma, double* out, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (num <= 0) return 0;
  const int total = cand_ptr[num];
  cudaError_t e = cudaSuccess;
  if (g.cand_ptr_cap < num + 1) {
    if (g.cand_ptr_d) cudaFree(g.cand_ptr_d);
    g.cand_ptr_d = nullptr;
    g.cand_ptr_cap = 0;
    e = cudaMalloc(&g.cand_ptr_d, sizeof(int32_t) * size_t(num + 1));
    if (e != cudaSuccess) return int(e);
    g.cand_ptr_cap = num + 1;
  }
  if (g.cand_cap < total) {   // float4 per candidate arc (saved records)
    if (g.cand_old) cudaFree(g.cand_old);
    g.cand_old = nullptr;
    g.cand_cap = 0;
    e = cudaMalloc(reinterpret_cast<void**>(&g.cand_old), sizeof(float4) * size_t(std::max(total, 1)));
    if (e != cudaSuccess) return int(e);
    g.cand_cap = total;
  }
  e = cudaMemcpyAsync(g.cand_ptr_d, cand_ptr, sizeof(int32_t) * size_t(num + 1), cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return int(e);
  SLParams P = sl_params(g);
  P.n_sigma = g.last_n_sigma;
  P.tau = g.last_tau;
  P.inv_tau = g.last_tau > 0.f ? 1.0 / double(g.last_tau) : 0.0;
  P.par = g.pass_fwd & 1u;
  P.stamp = g.inc_epoch + 1;
  g.inc_epoch += 2 * uint32_t(num);
  P.ep_blk = g.ep_blk;
  P.cand_ptr = g.cand_ptr_d;
  P.cand_arc = arc_ids;
  P.cand_m = reinterpret_cast<const float2*>(mean);
  P.cand_s = reinterpret_cast<const float2*>(sigma);
  P.cand_old = reinterpret_cast<float4*>(g.cand_old);
  P.cand_out = out;
  P.num_cand = num;
  if (!(g.last_tau > 0.f)) {   // hard mode: undo log instead of a second cone pass per candidate
    if (!g.elog) {
      const int cap = std::max(1024, std::min(g.num_heads, 1 << 20));
      e = cudaMalloc(&g.elog, sizeof(EvLog) * size_t(cap) + sizeof(int2) * size_t(cap) + 16);
      if (e != cudaSuccess) return int(e);
      g.elog_cap = cap;
    }
    P.elog = reinterpret_cast<EvLog*>(g.elog);
    P.flog = reinterpret_cast<int2*>(P.elog + g.elog_cap);
    P.elog_n = reinterpret_cast<uint32_t*>(P.flog + g.elog_cap);
    P.elog_cap = g.elog_cap;
  }
  const bool lse = g.last_tau > 0.f;
  const int err = launch_coop(lse ? (const void*)eval_kernel<true> : (const void*)eval_kernel<false>, g.sl_grid,
                              kSLFwdThreads, kEvalSmem, P, st, "eval");
  g.folded_valid = false;
  return err;
}

int launch_backward_sl(DevGraph& g, float* d_arc_mean, float* d_src, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (g.n == 0) return 0;
  SLParams P = sl_params(g);
  P.d_mean = d_arc_mean;
  P.d_src = d_src;
  if (g.bsnap_req) {   // snapshot for insta_backward_update
    P.acc_b = g.acc_b;
    P.hab_b = g.hab_b;
  }
  const bool lse = g.last_tau > 0.f;
  return launch_coop(lse ? (const void*)bwdl_kernel<true> : (const void*)bwdl_kernel<false>, g.sl_grid_b,
                     kSLBwdThreads, kBStageBytes, P, st, lse ? "bwd_lse" : "bwd");
}

// insta_backward_update: a snapshot backward (full sweep backward + snapshot), or the
// incremental update from the snapshot (seeds, diff of the touched heads, reverse cone)
int launch_backward_update(DevGraph& g, float* d_arc_mean, bool full, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (g.n == 0) return 0;
  const bool lse = g.last_tau > 0.f;
  const size_t H = size_t(std::max(g.num_heads, 1)), X = size_t(std::max<int64_t>(g.num_ext, 1));
  cudaError_t e = cudaSuccess;
  if (!g.acc_b) {   // snapshot arrays, allocated on first use
    e = cudaMalloc(&g.acc_b, sizeof(long long) * 2 * H);
    if (e == cudaSuccess) e = cudaMalloc(&g.hab_b, sizeof(float2) * H);
    if (e == cudaSuccess) e = cudaMalloc(&g.hseed_b, sizeof(float2) * H);
    if (e == cudaSuccess) e = cudaMalloc(&g.hwin_b, sizeof(int32_t) * H);
    if (e == cudaSuccess) e = cudaMalloc(&g.fwin_b, sizeof(int32_t) * X);
    if (e == cudaSuccess) e = cudaMalloc(&g.ew_b, sizeof(float4) * X);
    if (e == cudaSuccess) e = cudaMalloc(&g.efw_b, sizeof(float4) * X);
    if (e == cudaSuccess) e = cudaMalloc(&g.btouch, sizeof(uint32_t) * H);
    if (e == cudaSuccess) e = cudaMalloc(&g.bdirty, sizeof(uint32_t) * H);
    if (e == cudaSuccess) e = cudaMalloc(&g.bl_cnt, sizeof(uint32_t) * size_t(std::max(g.num_slevels, 1)));
    if (e == cudaSuccess) e = cudaMemsetAsync(g.btouch, 0, sizeof(uint32_t) * H, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(g.bdirty, 0, sizeof(uint32_t) * H, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(g.bl_cnt, 0, sizeof(uint32_t) * size_t(std::max(g.num_slevels, 1)), st);
    if (e != cudaSuccess) return int(e);
  }
  SLParams P = sl_params(g);
  P.d_mean = d_arc_mean;
  P.acc_b = g.acc_b;
  P.hab_b = g.hab_b;
  P.hseed_b = g.hseed_b;
  P.hwin_b = g.hwin_b;
  P.fwin_b = g.fwin_b;
  P.ew_b = g.ew_b;
  P.efw_b = g.efw_b;
  P.btouch = g.btouch;
  P.bepoch = g.bepoch;
  P.bdirty = g.bdirty;
  P.bl_cnt = g.bl_cnt;
  P.bstamp = ++g.bstamp;
  if (full) {   // the full backward (seeds, zero fills, sweep) writing acc_b / hab_b, then weights and seeds
    g.bsnap_req = true;
    int err = launch_backward(g, nullptr, d_arc_mean, nullptr, nullptr, stream);
    g.bsnap_req = false;
    if (err) return err;
    e = cudaMemcpyAsync(g.hseed_b, g.hseed, sizeof(float2) * H, cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess && !lse) e = cudaMemcpyAsync(g.hwin_b, g.hwin, sizeof(int32_t) * H, cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess && !lse) e = cudaMemcpyAsync(g.fwin_b, g.fwin, sizeof(int32_t) * X, cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess && lse) e = cudaMemcpyAsync(g.ew_b, g.ew, sizeof(float4) * X, cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess && lse) e = cudaMemcpyAsync(g.efw_b, g.efw, sizeof(float4) * X, cudaMemcpyDeviceToDevice, st);
    g.binc_heads = g.num_heads;
  } else {
    e = cudaMemsetAsync(g.counters + 2, 0, sizeof(unsigned long long), st);
    if (e != cudaSuccess) return int(e);
    int err = launch_seeds(g, stream);   // endpoint seeds from the current slacks (TNS)
    if (err) return err;
    const int blocks = int(std::min<size_t>((H + 255) / 256, size_t(std::max(g.sl_grid, 1)) * 8));
    if (lse) bdiff_kernel<true><<<blocks, 256, 0, st>>>(P);
    else bdiff_kernel<false><<<blocks, 256, 0, st>>>(P);
    err = int(cudaGetLastError());
    if (err) return err;
    err = launch_coop(lse ? (const void*)bwdi_kernel<true> : (const void*)bwdi_kernel<false>, g.sl_grid_b,
                      kSLBwdThreads, 0, P, st, "bwdi");
    if (err) return err;
  }
  ++g.bepoch;   // heads touched from now on differ from this snapshot
  return int(e);
}

int launch_fold_fill(DevGraph& g, void* stream) {
  if (g.folded_valid || g.num_ext == 0) return 0;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  SLParams P = sl_params(g);
  P.n_sigma = g.last_n_sigma;
  P.tau = g.last_tau;
  P.inv_tau = g.last_tau > 0.f ? 1.0 / double(g.last_tau) : 0.0;
  P.par = g.pass_fwd & 1u;
  const int blocks = int((g.num_ext + 255) / 256);
  if (g.last_tau > 0.f) fold_fill_kernel<true><<<blocks, 256, 0, st>>>(P, g.num_ext);
  else fold_fill_kernel<false><<<blocks, 256, 0, st>>>(P, g.num_ext);
  const int err = int(cudaGetLastError());
  if (!err) g.folded_valid = true;
  return err;
}

}  // namespace insta
