// device_common.cuh -- PTX helpers shared by the single-scenario (kernels.cu)
// and batched (batch.cu) propagation kernels: memory-model accesses, the
// parity-tagged words of the dataflow synchronization, mbarrier + TMA bulk
// copies, and the per-candidate primitives of Eq 1-3.
#pragma once
#include <cuda_runtime.h>

// Back-off between re-polls of a dataflow word that is not ready yet (ns;
// 0 = spin without sleeping).  Measured on B200 at C4: 0 / 5 / 20 / 100 ns give the same fwd (0.578 ms)
// and bwd (0.605 ms) times within noise -- the wait is for the producer, not the poll period.
#ifndef INSTA_POLL_NS
#define INSTA_POLL_NS 20
#endif
#if INSTA_POLL_NS > 0
#define INSTA_POLL_SLEEP() __nanosleep(INSTA_POLL_NS)
#else
#define INSTA_POLL_SLEEP() ((void)0)
#endif

#include <cstdint>

namespace insta {

// Dataflow waits are bounded: a word that never arrives (which valid inputs
// cannot cause; insta_backward / insta_forward_batch validate the adjoint
// bound of the count-folded accumulators) aborts the kernel -- the launch
// fails with an error -- instead of hanging the GPU.
#ifndef INSTA_POLL_LIMIT
#define INSTA_POLL_LIMIT (1u << 26)
#endif
__device__ __forceinline__ void insta_poll_pause(uint32_t& n) {
  INSTA_POLL_SLEEP();
  if (++n > INSTA_POLL_LIMIT) __trap();
}

constexpr int kUnateShiftC = 30;   // fin_src bits 30..31: unateness (internal.h kUnateShift)

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

// ---- parity-tagged words ----
__device__ __forceinline__ double with_par(double x, uint32_t par) {
  return __longlong_as_double((__double_as_longlong(x) & ~1ll) | (long long)par);
}
__device__ __forceinline__ double strip(unsigned long long b) { return __longlong_as_double((long long)(b & ~1ull)); }
// The var_F word (last word) of a pin record also carries, in bit 1, the
// "record changed in this pass" flag of the incremental pass; its value is used
// with both low bits cleared (identically in every kernel).
__device__ __forceinline__ double with_tag(double x, uint32_t par, uint32_t chg) {
  return __longlong_as_double((__double_as_longlong(x) & ~3ll) | (long long)(par | (chg << 1)));
}
__device__ __forceinline__ double strip2(unsigned long long b) { return __longlong_as_double((long long)(b & ~3ull)); }
__device__ __forceinline__ uint32_t tag_changed(unsigned long long d) { return uint32_t(d >> 1) & 1u; }
__device__ __forceinline__ float with_parf(float x, uint32_t par) {
  return __uint_as_float((__float_as_uint(x) & ~1u) | par);
}
__device__ __forceinline__ float stripf(uint32_t b) { return __uint_as_float(b & ~1u); }

__device__ __forceinline__ void ld2_u64(const void* p, unsigned long long& a, unsigned long long& b) {
  asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ void st2_u64(void* p, double a, double b) {
  asm volatile("st.relaxed.gpu.global.v2.f64 [%0], {%1, %2};" ::"l"(p), "d"(a), "d"(b) : "memory");
}
__device__ __forceinline__ void ld2_u32(const void* p, uint32_t& a, uint32_t& b) {
  asm volatile("ld.relaxed.gpu.global.v2.b32 {%0, %1}, [%2];" : "=r"(a), "=r"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ void st2_f32(void* p, float a, float b) {
  asm volatile("st.relaxed.gpu.global.v2.f32 [%0], {%1, %2};" ::"l"(p), "f"(a), "f"(b) : "memory");
}

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, 1000000;\n\t"   // suspend, don't spin
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

// sigma = sqrt(var) for the corner arrival: the hardware square root
// (sqrt.approx.f32, ~1 ulp; deterministic) of the fp32-rounded variance.
__device__ __forceinline__ float sigma_of(double var) {
  float r;
  asm("sqrt.approx.f32 %0, %1;" : "=f"(r) : "f"(float(var)));
  return r;
}

// source transitions of an arc for sink transition rf: POS {rf}; NEG {~rf}
// (Alg 1 l.8); NON (rf, ~rf) (reading R3).
__device__ __forceinline__ int n_src_tr(int u) { return u == 2 ? 2 : 1; }
__device__ __forceinline__ int src_tr(int rf, int u, int a) { return (u == 1 || a == 1) ? (rf ^ 1) : rf; }

// --------------------------------------------------------------------------
// Eq 1-3 for one candidate: arc e = (j -> i), sink transition rf, source
// transition s.  State carries the variance (Eq 2 is additive in it):
//   mu_c  = mu_j[s] + arc_mean[rf]                 (Eq 1, Alg 1 l.12)
//   var_c = var_j[s] + arc_std[rf]^2               (Eq 2, Alg 1 l.13)
//   A_c   = mu_c + n_sigma * sqrt(var_c)           (Eq 3, Alg 1 l.14)
// mean and variance accumulate in fp64; the sqrt of the corner is fp32.
// --------------------------------------------------------------------------
struct Gath {
  double mu0, mu1, v0, v1;
};

struct Cand {
  double mu, var, A;
  float sig;
};


// Pin state words as loaded (parity bits still in place).
struct Raw {
  unsigned long long a, b, c, d;
};

// one 256-bit access per 32-byte pin record (LDG/STG .256 on sm_100a)
__device__ __forceinline__ bool raw_ready(const Raw& r, uint32_t par) {
  return (((r.a & r.b & r.c & r.d) & 1ull) == par) && (((r.a | r.b | r.c | r.d) & 1ull) == par);
}

__device__ __forceinline__ Gath unpack(const Raw& r) {
  Gath g;
  g.mu0 = strip(r.a);
  g.mu1 = strip(r.b);
  g.v0 = strip(r.c);
  g.v1 = strip2(r.d);
  return g;
}

__device__ __forceinline__ Cand make_cand(const Gath& st, const float4& ms, int rf, int s, double ns) {
  const double se = double(rf ? ms.w : ms.z);
  Cand c;
  c.mu = (s ? st.mu1 : st.mu0) + double(rf ? ms.y : ms.x);
  c.var = (s ? st.v1 : st.v0) + se * se;
  c.sig = sigma_of(c.var);
  c.A = c.mu + ns * double(c.sig);
  return c;
}


// Merge of one (pin, rf): first arg-max (strict ">"), LSE normalizer.
struct Merge {
  double best, mu, var;
  float sig, sum;
  int k, s;
};

__device__ __forceinline__ void merge_init(Merge& m) {
  m.best = 0.0;
  m.mu = 0.0;
  m.var = 0.0;
  m.sig = 0.f;
  m.sum = 0.f;
  m.k = -1;
  m.s = 0;
}

__device__ __forceinline__ void merge_max(Merge& m, const Cand& c, int k, int s) {
  if (m.k < 0 || c.A > m.best) {   // Alg 2 l.4: replace only if strictly greater
    m.best = c.A;
    m.mu = c.mu;
    m.var = c.var;
    m.sig = c.sig;
    m.k = k;
    m.s = s;
  }
}

// Eq 6 weight of a candidate given its merge (LSE)
__device__ __forceinline__ float lse_term(const Cand& c, const Merge& m, double tau) {
  return expf(float((c.A - m.best) * tau));   // tau: the inverse temperature 1/tau
}

// Merge of one (pin, rf) over its candidates in canonical order (fanin row,
// then s = rf before ~rf): Alg 1 / Alg 2 with K = 1 (first arg-max, strict
// ">") or Eq 4 (LSE with M = the arg-max).  Only corner arrivals are compared;
// the winner's distribution is re-evaluated once (bit-identical to its scan
// value).  arc(k, w, ms, raw) yields arc k's source word, (scenario) arc record
// and gathered source words.  Shared by the single-scenario, incremental and
// batched kernels.
struct RfOut {
  double mu, var, best;
  float sum, sig;
  int win;   // arg-max: k | s << 15
};

// exp((A - M) / tau) for the LSE normalizer and Eq 6 weights: fp32 exponent
// (hardware ex2, deterministic), argument formed in fp64.
__device__ __forceinline__ float lse_w(double A, double best, double inv_tau) {
  return __expf(float((A - best) * inv_tau));
}

// LSE arrival (Eq 4): M + tau * log(sum)
__device__ __forceinline__ double lse_arrival(double best, double tau, float sum) {
  return best + tau * double(__logf(sum));
}

template <bool kLSE, class ArcFn>
__device__ __forceinline__ RfOut merge_rf(double ns, double tau, double inv_tau, int rf, int nf, ArcFn&& arc) {
  double best = 0.0;
  int bk = -1, bs = 0;
  for (int k = 0; k < nf; ++k) {
    int32_t w;
    float4 ms;
    Raw r;
    arc(k, w, ms, r);
    const Gath st = unpack(r);
    const int u = int(uint32_t(w) >> kUnateShiftC);
    const int s0 = src_tr(rf, u, 0);
    const double a0 = make_cand(st, ms, rf, s0, ns).A;
    if (bk < 0 || a0 > best) {   // Alg 2 l.4: replace only if strictly greater
      best = a0;
      bk = k;
      bs = s0;
    }
    if (u == 2) {
      const double a1 = make_cand(st, ms, rf, rf ^ 1, ns).A;
      if (a1 > best) {
        best = a1;
        bk = k;
        bs = rf ^ 1;
      }
    }
  }
  RfOut o;
  {
    int32_t w;
    float4 ms;
    Raw r;
    arc(bk, w, ms, r);
    const Cand c = make_cand(unpack(r), ms, rf, bs, ns);   // the winner (Alg 1 l.15)
    o.mu = c.mu;
    o.var = c.var;
    o.sig = c.sig;
  }
  o.best = best;
  o.win = bk | (bs << 15);
  o.sum = 0.f;
  if (kLSE) {
    // Eq 4: A_i = M + tau * log(sum_c exp((A_c - M) / tau)); reading R1:
    // sigma_i = sigma of the arg-max, mu_i = A_i - n_sigma * sigma_i.
    float sum = 0.f;
    for (int k = 0; k < nf; ++k) {
      int32_t w;
      float4 ms;
      Raw r;
      arc(k, w, ms, r);
      const Gath st = unpack(r);
      const int u = int(uint32_t(w) >> kUnateShiftC);
      sum += lse_w(make_cand(st, ms, rf, src_tr(rf, u, 0), ns).A, best, inv_tau);
      if (u == 2) sum += lse_w(make_cand(st, ms, rf, rf ^ 1, ns).A, best, inv_tau);
    }
    o.sum = sum;
    o.mu = lse_arrival(best, tau, sum) - ns * double(o.sig);
  }
  return o;
}

// merge_rf for nf <= NMAX with the candidate loop unrolled (arc(k) is called
// with compile-time k, so register-held source words need no run-time
// selection) and the winner kept from the scan instead of re-evaluated: the
// same operations in the same order as merge_rf, hence bit-identical.
template <bool kLSE, int NMAX, class ArcFn>
__device__ __forceinline__ RfOut merge_rf_unrolled(double ns, double tau, double inv_tau, int rf, int nf, ArcFn&& arc) {
  double best = 0.0;
  int bk = -1, bs = 0;
  Cand win;
  win.mu = win.var = win.A = 0.0;
  win.sig = 0.f;
#pragma unroll
  for (int k = 0; k < NMAX; ++k) {
    if (k < nf) {
      int32_t w;
      float4 ms;
      Raw r;
      arc(k, w, ms, r);
      const Gath st = unpack(r);
      const int u = int(uint32_t(w) >> kUnateShiftC);
      const int s0 = src_tr(rf, u, 0);
      const Cand c0 = make_cand(st, ms, rf, s0, ns);
      if (bk < 0 || c0.A > best) {   // Alg 2 l.4: replace only if strictly greater
        best = c0.A;
        bk = k;
        bs = s0;
        win = c0;
      }
      if (u == 2) {
        const Cand c1 = make_cand(st, ms, rf, rf ^ 1, ns);
        if (c1.A > best) {
          best = c1.A;
          bk = k;
          bs = rf ^ 1;
          win = c1;
        }
      }
    }
  }
  RfOut o;
  o.mu = win.mu;
  o.var = win.var;
  o.sig = win.sig;
  o.best = best;
  o.win = bk | (bs << 15);
  o.sum = 0.f;
  if (kLSE) {
    float sum = 0.f;
#pragma unroll
    for (int k = 0; k < NMAX; ++k) {
      if (k < nf) {
        int32_t w;
        float4 ms;
        Raw r;
        arc(k, w, ms, r);
        const Gath st = unpack(r);
        const int u = int(uint32_t(w) >> kUnateShiftC);
        sum += lse_w(make_cand(st, ms, rf, src_tr(rf, u, 0), ns).A, best, inv_tau);
        if (u == 2) sum += lse_w(make_cand(st, ms, rf, rf ^ 1, ns).A, best, inv_tau);
      }
    }
    o.sum = sum;
    o.mu = lse_arrival(best, tau, sum) - ns * double(o.sig);
  }
  return o;
}

// Merge of a pin with exactly one fanin arc (source words st, unateness u,
// record ms): the same operation sequence as merge_rf with nf = 1 -- scan
// (a0, then a1 for a non-unate arc, strict ">"), winner, LSE sum 0 + w0
// (+ w1), Eq 4 arrival, Eq 6 weights -- with each candidate evaluated once;
// hard mode with a unate arc has a single candidate, so its corner (and square
// root) is not needed.  Bit-identical to merge_rf + arc_weights (nf = 1).
struct Merge1 {
  double mu[2], var[2];
  int32_t win;   // arg-max word {R: s << 15, F: << 16}
  float4 wt;     // Eq 6 weights {w[R][R], w[R][F], w[F][R], w[F][F]} (LSE)
  __device__ __forceinline__ Raw stored(uint32_t par) const {   // the words a store with parity writes
    Raw o;
    o.a = (unsigned long long)__double_as_longlong(with_par(mu[0], par));
    o.b = (unsigned long long)__double_as_longlong(with_par(mu[1], par));
    o.c = (unsigned long long)__double_as_longlong(with_par(var[0], par));
    o.d = (unsigned long long)__double_as_longlong(with_tag(var[1], par, 0u));
    return o;
  }
};

template <bool kLSE>
__device__ __forceinline__ void merge1(const Gath& st, int u, const float4& ms, double ns, double tau, double inv_tau,
                                       Merge1& m) {
  int win[2];
  float wt[2][2] = {{0.f, 0.f}, {0.f, 0.f}};
#pragma unroll
  for (int rf = 0; rf < 2; ++rf) {
    const int s0 = src_tr(rf, u, 0);
    if (!kLSE && u != 2) {
      const double se = double(rf ? ms.w : ms.z);
      m.mu[rf] = (s0 ? st.mu1 : st.mu0) + double(rf ? ms.y : ms.x);   // = make_cand(...).mu
      m.var[rf] = (s0 ? st.v1 : st.v0) + se * se;                       // = make_cand(...).var
      win[rf] = s0 << 15;
      continue;
    }
    const Cand c0 = make_cand(st, ms, rf, s0, ns);
    Cand cb = c0;
    int bs = s0;
    Cand c1 = c0;
    if (u == 2) {
      c1 = make_cand(st, ms, rf, rf ^ 1, ns);
      if (c1.A > c0.A) {
        cb = c1;
        bs = rf ^ 1;
      }
    }
    m.mu[rf] = cb.mu;
    m.var[rf] = cb.var;
    win[rf] = bs << 15;
    if (kLSE && u != 2) {
      // one candidate: w0 = exp(0) = 1 and the normalizer is 0 + 1 = 1 exactly,
      // ln(1) = 0, 1 / 1 = 1: the Eq 4 arrival is A_c itself and the Eq 6
      // weight is 1 (the same values the general sequence below produces)
      m.mu[rf] = (cb.A + 0.0) - ns * double(cb.sig);
      wt[rf][s0] = 1.f;
    } else if (kLSE) {
      float sum = 0.f;
      const float w0 = lse_w(c0.A, cb.A, inv_tau);
      sum += w0;
      float w1 = 0.f;
      if (u == 2) {
        w1 = lse_w(c1.A, cb.A, inv_tau);
        sum += w1;
      }
      m.mu[rf] = lse_arrival(cb.A, tau, sum) - ns * double(cb.sig);
      const float inv_sum = 1.f / sum;
      wt[rf][s0] = w0 * inv_sum;
      if (u == 2) wt[rf][rf ^ 1] = w1 * inv_sum;
    }
  }
  m.win = win[0] | (win[1] << 16);
  m.wt = make_float4(wt[0][0], wt[0][1], wt[1][0], wt[1][1]);
}

// Eq 6 weights {w[rf][s=R], w[rf][s=F]} of arc k's candidates for transition rf
template <class ArcFn>
__device__ __forceinline__ float2 arc_weights(double ns, double inv_tau, int rf, int k, const RfOut& o,
                                              ArcFn&& arc) {
  int32_t w;
  float4 ms;
  Raw r;
  arc(k, w, ms, r);
  const Gath st = unpack(r);
  const int u = int(uint32_t(w) >> kUnateShiftC);
  float wt[2] = {0.f, 0.f};
  const int s0 = src_tr(rf, u, 0);
  const float inv_sum = 1.f / o.sum;
  wt[s0] = lse_w(make_cand(st, ms, rf, s0, ns).A, o.best, inv_tau) * inv_sum;
  if (u == 2) wt[rf ^ 1] = lse_w(make_cand(st, ms, rf, rf ^ 1, ns).A, o.best, inv_tau) * inv_sum;
  return make_float2(wt[0], wt[1]);
}

}  // namespace insta
