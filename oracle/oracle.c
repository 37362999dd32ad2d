/*
 * oracle.c -- plain, slow, obviously-correct fp64 CPU oracle of INSTA's K=1
 * statistical arrival propagation, endpoint slack / WNS / TNS and the TNS
 * backward (PAPER.md, "INSTA", DAC'25).
 *
 * TEST INFRASTRUCTURE, NOT PRODUCT.  Loaded only by tests/, by
 * __graft_entry__.smoke() and by bench.py's cpu_baseline / --impl reference
 * legs.  Shares nothing with the CUDA path.
 *
 * Notation follows the paper: arrival_mean (mu), arrival_std (sigma) and the
 * corner arrival A = mu + N_sigma * sigma (Eq 1-3); arc delays are
 * indexed by the sink transition rf (Alg 1 l.12-13); the source
 * transition is ~rf for negative-unate arcs (Alg 1 l.8).  The merge is
 * Alg 1/Alg 2 with K = 1 ("hard", strict ">" P:L97, L115) or the LSE operator
 * (Eq 4) with softmax gradients (Eq 6).
 *
 * Parity status of each function (DESIGN.md §3 "pins"):
 *   orc_levelize   pinned (networkx.topological_generations, invariants)
 *   orc_forward    hard: pinned (brute-force max path for sigma==0; traced
 *                  critical-path identity for sigma>0; hand-worked example)
 *                  lse, sigma==0: pinned (tau*logsumexp over all paths)
 *                  lse, sigma>0: PARITY UNPINNED w.r.t. paper intent (reading
 *                  #1: sigma of the merged arrival = sigma of the arg-max;
 *                  pinned only by limits tau->0 / sigma->0, FD consistency and
 *                  the equal-variance layered closed form, which holds for
 *                  any choice of the kept sigma)
 *   orc_slack      pinned (closed forms)
 *   orc_backward   pinned (central finite differences of orc_forward; path
 *                  marginals for sigma==0 LSE; integer path counts in hard mode)
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

enum { RISE = 0, FALL = 1 };
enum { U_POS = 0, U_NEG = 1, U_NON = 2 };

/* ------------------------------------------------------------------------- */
/* O1: validation (C ABI error rules)                           */
/* ------------------------------------------------------------------------- */
static int finite(double x) { return isfinite(x); }

int orc_validate(const orc_graph* g, double n_sigma, double tau) {
  if (!g || g->num_pins < 0 || g->num_arcs < 0 || g->num_endpoints < 0) return 1;
  if (!finite(n_sigma) || n_sigma < 0 || !finite(tau) || tau < 0) return 1;
  if (g->num_arcs > 0 && (!g->arc_from || !g->arc_to || !g->arc_unate || !g->arc_mean || !g->arc_sigma))
    return 1;
  for (int64_t e = 0; e < g->num_arcs; ++e) {
    if (g->arc_from[e] < 0 || g->arc_from[e] >= g->num_pins) return 1;
    if (g->arc_to[e] < 0 || g->arc_to[e] >= g->num_pins) return 1;
    if (g->arc_unate[e] > U_NON) return 1;
    for (int rf = 0; rf < 2; ++rf) {
      if (!finite(g->arc_mean[2 * e + rf]) || !finite(g->arc_sigma[2 * e + rf])) return 1;
      if (g->arc_sigma[2 * e + rf] < 0) return 1;
    }
  }
  for (int64_t p = 0; p < 2 * (int64_t)g->num_pins; ++p) {
    if (g->src_mean && !finite(g->src_mean[p])) return 1;
    if (g->src_sigma && (!finite(g->src_sigma[p]) || g->src_sigma[p] < 0)) return 1;
  }
  if (g->num_endpoints > 0 && (!g->ep_pin || !g->ep_rat)) return 1;
  char* seen = calloc((size_t)g->num_pins + 1, 1);
  for (int32_t k = 0; k < g->num_endpoints; ++k) {
    int32_t p = g->ep_pin[k];
    if (p < 0 || p >= g->num_pins || seen[p]) { free(seen); return 1; }
    seen[p] = 1;
    if (!finite(g->ep_rat[2 * k]) || !finite(g->ep_rat[2 * k + 1])) { free(seen); return 1; }
  }
  free(seen);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* O2: levelization by topological sort ("constructs and levelizes its  */
/* timing graph ... pins within the same level are processed independently") */
/* level(p) = 0 if indeg(p) = 0, else 1 + max level of its fanin sources.     */
/* ------------------------------------------------------------------------- */
typedef struct {
  int32_t n, num_levels;
  int64_t e;
  int32_t *level, *order, *pos;         /* pos[p] = canonical position of pin p */
  int32_t *fanin_ptr, *fanin_arc;       /* over canonical positions            */
  int32_t *fanout_ptr, *fanout_arc;
  int32_t *level_ptr;                   /* [num_levels + 1] canonical range of each level */
} topo_t;

static void topo_free(topo_t* t) {
  free(t->level); free(t->order); free(t->pos);
  free(t->fanin_ptr); free(t->fanin_arc); free(t->fanout_ptr); free(t->fanout_arc);
  free(t->level_ptr);
  memset(t, 0, sizeof *t);
}

/* returns 0 ok, 2 cycle */
static int topo_build(int32_t n, int64_t E, const int32_t* from, const int32_t* to, topo_t* t) {
  memset(t, 0, sizeof *t);
  t->n = n; t->e = E;
  t->level = calloc((size_t)n + 1, sizeof(int32_t));
  t->order = calloc((size_t)n + 1, sizeof(int32_t));
  t->pos = calloc((size_t)n + 1, sizeof(int32_t));
  t->fanin_ptr = calloc((size_t)n + 1, sizeof(int32_t));
  t->fanout_ptr = calloc((size_t)n + 1, sizeof(int32_t));
  t->fanin_arc = calloc((size_t)E + 1, sizeof(int32_t));
  t->fanout_arc = calloc((size_t)E + 1, sizeof(int32_t));

  /* caller-indexed out-adjacency (arcs of each pin, ascending arc id) */
  int32_t* out_ptr = calloc((size_t)n + 1, sizeof(int32_t));
  int32_t* out_arc = calloc((size_t)E + 1, sizeof(int32_t));
  int32_t* indeg = calloc((size_t)n + 1, sizeof(int32_t));
  for (int64_t e = 0; e < E; ++e) { out_ptr[from[e] + 1]++; indeg[to[e]]++; }
  for (int32_t p = 0; p < n; ++p) out_ptr[p + 1] += out_ptr[p];
  int32_t* fill = calloc((size_t)n + 1, sizeof(int32_t));
  for (int64_t e = 0; e < E; ++e) out_arc[out_ptr[from[e]] + fill[from[e]]++] = (int32_t)e;

  /* Kahn's algorithm with explicit levels */
  int32_t* queue = malloc(((size_t)n + 1) * sizeof(int32_t));
  int32_t head = 0, tail = 0;
  for (int32_t p = 0; p < n; ++p) if (indeg[p] == 0) { queue[tail++] = p; t->level[p] = 0; }
  while (head < tail) {
    int32_t p = queue[head++];
    for (int32_t k = out_ptr[p]; k < out_ptr[p + 1]; ++k) {
      int32_t q = to[out_arc[k]];
      if (t->level[p] + 1 > t->level[q]) t->level[q] = t->level[p] + 1;
      if (--indeg[q] == 0) queue[tail++] = q;
    }
  }
  int cyc = (tail < n);
  free(queue); free(indeg); free(fill); free(out_ptr); free(out_arc);
  if (cyc) { topo_free(t); return 2; }

  /* canonical order: pins sorted by (level, pin id) -- counting sort by level */
  int32_t L = 0;
  for (int32_t p = 0; p < n; ++p) if (t->level[p] + 1 > L) L = t->level[p] + 1;
  t->num_levels = L;
  int32_t* cnt = calloc((size_t)L + 1, sizeof(int32_t));
  for (int32_t p = 0; p < n; ++p) cnt[t->level[p] + 1]++;
  for (int32_t l = 0; l < L; ++l) cnt[l + 1] += cnt[l];
  t->level_ptr = calloc((size_t)L + 2, sizeof(int32_t));
  for (int32_t l = 0; l <= L; ++l) t->level_ptr[l] = cnt[l];
  for (int32_t p = 0; p < n; ++p) { int32_t k = cnt[t->level[p]]++; t->order[k] = p; t->pos[p] = k; }
  free(cnt);

  /* fanin / fanout rows in canonical order, arcs ascending by caller arc id */
  for (int64_t e = 0; e < E; ++e) { t->fanin_ptr[t->pos[to[e]] + 1]++; t->fanout_ptr[t->pos[from[e]] + 1]++; }
  for (int32_t k = 0; k < n; ++k) { t->fanin_ptr[k + 1] += t->fanin_ptr[k]; t->fanout_ptr[k + 1] += t->fanout_ptr[k]; }
  int32_t* fi = calloc((size_t)n + 1, sizeof(int32_t));
  int32_t* fo = calloc((size_t)n + 1, sizeof(int32_t));
  for (int64_t e = 0; e < E; ++e) {
    int32_t a = t->pos[to[e]], b = t->pos[from[e]];
    t->fanin_arc[t->fanin_ptr[a] + fi[a]++] = (int32_t)e;
    t->fanout_arc[t->fanout_ptr[b] + fo[b]++] = (int32_t)e;
  }
  free(fi); free(fo);
  return 0;
}

int orc_levelize(int32_t num_pins, int64_t num_arcs, const int32_t* arc_from,
                 const int32_t* arc_to, int32_t* level, int32_t* order,
                 int32_t* fanin_ptr, int32_t* fanin_arc, int32_t* fanout_ptr,
                 int32_t* fanout_arc, int32_t* num_levels) {
  if (num_pins < 0 || num_arcs < 0 || num_arcs >= ((int64_t)1 << 31)) return 1;
  for (int64_t e = 0; e < num_arcs; ++e)
    if (arc_from[e] < 0 || arc_from[e] >= num_pins || arc_to[e] < 0 || arc_to[e] >= num_pins) return 1;
  topo_t t;
  int st = topo_build(num_pins, num_arcs, arc_from, arc_to, &t);
  if (st) return st;
  if (level) memcpy(level, t.level, sizeof(int32_t) * (size_t)num_pins);
  if (order) memcpy(order, t.order, sizeof(int32_t) * (size_t)num_pins);
  if (fanin_ptr) memcpy(fanin_ptr, t.fanin_ptr, sizeof(int32_t) * ((size_t)num_pins + 1));
  if (fanout_ptr) memcpy(fanout_ptr, t.fanout_ptr, sizeof(int32_t) * ((size_t)num_pins + 1));
  if (fanin_arc) memcpy(fanin_arc, t.fanin_arc, sizeof(int32_t) * (size_t)num_arcs);
  if (fanout_arc) memcpy(fanout_arc, t.fanout_arc, sizeof(int32_t) * (size_t)num_arcs);
  if (num_levels) *num_levels = t.num_levels;
  topo_free(&t);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* O4: candidates of (pin i, sink transition rf)                              */
/* For each fanin arc e = (j -> i) in row order and each source transition    */
/* s in S(rf, U[e]) -- POS: {rf}; NEG: {~rf} (Alg 1 l.8); NON: (rf, ~rf):      */
/*   mean  mu_c  = mu_j[s] + arc_mean[e][rf]                 (Eq 1, Alg 1 l.12) */
/*   std   sig_c = sqrt(sig_j[s]^2 + arc_std[e][rf]^2)       (Eq 2, Alg 1 l.13) */
/*   arrival A_c = mu_c + N_sigma * sig_c                    (Eq 3, Alg 1 l.14) */
/* ------------------------------------------------------------------------- */
typedef struct { int32_t arc, src; int s; double mu, sig, A; } cand_t;

static int sources_of(int rf, int unate, int* s_out) {
  if (unate == U_POS) { s_out[0] = rf; return 1; }
  if (unate == U_NEG) { s_out[0] = 1 - rf; return 1; }
  s_out[0] = rf; s_out[1] = 1 - rf; return 2;
}

static int candidates(const orc_graph* g, const topo_t* t, int32_t k /*canonical pos*/, int rf,
                      double n_sigma, const double* mu, const double* sig, cand_t* c) {
  int n = 0;
  for (int32_t q = t->fanin_ptr[k]; q < t->fanin_ptr[k + 1]; ++q) {
    int32_t e = t->fanin_arc[q];
    int32_t j = g->arc_from[e];
    int ss[2];
    int ns = sources_of(rf, g->arc_unate[e], ss);
    for (int a = 0; a < ns; ++a) {
      int s = ss[a];
      double arc_mean = g->arc_mean[2 * (int64_t)e + rf];
      double arc_std = g->arc_sigma[2 * (int64_t)e + rf];
      c[n].arc = e; c[n].src = j; c[n].s = s;
      c[n].mu = mu[2 * (int64_t)j + s] + arc_mean;
      c[n].sig = sqrt(sig[2 * (int64_t)j + s] * sig[2 * (int64_t)j + s] + arc_std * arc_std);
      c[n].A = c[n].mu + n_sigma * c[n].sig;
      ++n;
    }
  }
  return n;
}

/* first arg-max: a later candidate replaces only if strictly greater (Alg 2 l.4) */
static int first_argmax(const cand_t* c, int n) {
  int best = 0;
  for (int a = 1; a < n; ++a) if (c[a].A > c[best].A) best = a;
  return best;
}

static int max_fanin(const topo_t* t) {
  int m = 1;
  for (int32_t k = 0; k < t->n; ++k) {
    int d = t->fanin_ptr[k + 1] - t->fanin_ptr[k];
    if (d > m) m = d;
  }
  return m;
}

/* O3 + O4 + O5 for the pin at canonical position k; mu/sig are the per-pin
 * state (Eq 1-2); c: candidate scratch. */
static void propagate_pin(const orc_graph* g, const topo_t* t, int32_t k, double n_sigma, double tau,
                          double* mu, double* sig, int32_t* win_arc, int8_t* win_s, double* gap, cand_t* c) {
  int32_t i = t->order[k];
  if (t->fanin_ptr[k] == t->fanin_ptr[k + 1]) {
    /* O3: startpoint -- clock arrival distribution, corner via Eq 3 */
    for (int rf = 0; rf < 2; ++rf) {
      mu[2 * (int64_t)i + rf] = g->src_mean ? g->src_mean[2 * (int64_t)i + rf] : 0.0;
      sig[2 * (int64_t)i + rf] = g->src_sigma ? g->src_sigma[2 * (int64_t)i + rf] : 0.0;
      if (win_arc) win_arc[2 * (int64_t)i + rf] = -1;
      if (win_s) win_s[2 * (int64_t)i + rf] = -1;
      if (gap) gap[2 * (int64_t)i + rf] = INFINITY;
    }
    return;
  }
  for (int rf = 0; rf < 2; ++rf) {
    int n = candidates(g, t, k, rf, n_sigma, mu, sig, c);
    int b = first_argmax(c, n);
    if (tau == 0.0) {
      /* hard: Alg 1 + Alg 2 with K = 1 -- keep the distribution of the max */
      mu[2 * (int64_t)i + rf] = c[b].mu;
      sig[2 * (int64_t)i + rf] = c[b].sig;
    } else {
      /* LSE (Eq 4): A_i = M + tau * log(sum exp((A_c - M)/tau)), M = max.
       * Reading #1: sigma_i = sigma of the arg-max; mu_i = A_i - N_sigma*sigma_i. */
      double M = c[b].A, sum = 0.0;
      for (int a = 0; a < n; ++a) sum += exp((c[a].A - M) / tau);
      double A_i = M + tau * log(sum);
      sig[2 * (int64_t)i + rf] = c[b].sig;
      mu[2 * (int64_t)i + rf] = A_i - n_sigma * c[b].sig;
    }
    if (win_arc) win_arc[2 * (int64_t)i + rf] = c[b].arc;
    if (win_s) win_s[2 * (int64_t)i + rf] = (int8_t)c[b].s;
    if (gap) {
      double second = -INFINITY;
      for (int a = 0; a < n; ++a) if (a != b && c[a].A > second) second = c[a].A;
      gap[2 * (int64_t)i + rf] = (n > 1) ? c[b].A - second : INFINITY;
    }
  }
}

/* Over the whole graph in canonical order.  The OpenMP build (liboracle_omp,
 * the bench's all-core CPU baseline) runs the pins of one level in parallel:
 * they only read earlier levels, so the result is the same. */
static void propagate(const orc_graph* g, const topo_t* t, double n_sigma, double tau,
                      double* mu, double* sig, int32_t* win_arc, int8_t* win_s, double* gap) {
#ifdef _OPENMP
  for (int32_t l = 0; l < t->num_levels; ++l) {
#pragma omp parallel
    {
      cand_t* c = malloc(sizeof(cand_t) * 2 * (size_t)max_fanin(t));
#pragma omp for schedule(static)
      for (int32_t k = t->level_ptr[l]; k < t->level_ptr[l + 1]; ++k)
        propagate_pin(g, t, k, n_sigma, tau, mu, sig, win_arc, win_s, gap, c);
      free(c);
    }
  }
#else
  cand_t* c = malloc(sizeof(cand_t) * 2 * (size_t)max_fanin(t));
  for (int32_t k = 0; k < t->n; ++k) propagate_pin(g, t, k, n_sigma, tau, mu, sig, win_arc, win_s, gap, c);
  free(c);
#endif
}

int orc_forward(const orc_graph* g, double n_sigma, double tau, double* A,
                double* sig, double* mu, int32_t* win_arc, int8_t* win_s,
                double* gap) {
  int st = orc_validate(g, n_sigma, tau);
  if (st) return st;
  topo_t t;
  st = topo_build(g->num_pins, g->num_arcs, g->arc_from, g->arc_to, &t);
  if (st) return st;
  size_t n2 = 2 * (size_t)g->num_pins + 2;
  double* m = malloc(n2 * sizeof(double));
  double* s = malloc(n2 * sizeof(double));
  propagate(g, &t, n_sigma, tau, m, s, win_arc, win_s, gap);
  for (int64_t p = 0; p < 2 * (int64_t)g->num_pins; ++p) {
    if (A) A[p] = m[p] + n_sigma * s[p];           /* Eq 3: the corner arrival */
    if (mu) mu[p] = m[p];
    if (sig) sig[p] = s[p];
  }
  free(m); free(s);
  topo_free(&t);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* O6: endpoint slack = RAT - A (setup), min over rf (tie -> R);              */
/* TNS = sum of min(0, slack) in endpoint order, WNS = min(0, min slack),     */
/* violations = #{slack < 0} (Table II signs P:L216-227).  */
/* ------------------------------------------------------------------------- */
int orc_slack(const orc_graph* g, const double* A, double* slack,
              uint8_t* rf_star, double* wns, double* tns, int32_t* num_viol) {
  double w = 0.0, t = 0.0;
  int32_t nv = 0;
  for (int32_t k = 0; k < g->num_endpoints; ++k) {
    int32_t p = g->ep_pin[k];
    double sr = g->ep_rat[2 * k + RISE] - A[2 * (int64_t)p + RISE];
    double sf = g->ep_rat[2 * k + FALL] - A[2 * (int64_t)p + FALL];
    int r = (sf < sr) ? FALL : RISE;
    double s = (r == FALL) ? sf : sr;
    if (slack) slack[k] = s;
    if (rf_star) rf_star[k] = (uint8_t)r;
    if (s < 0) { t += s; ++nv; }
    if (s < w) w = s;
  }
  if (wns) *wns = w;
  if (tns) *tns = t;
  if (num_viol) *num_viol = nv;
  return 0;
}

/* ------------------------------------------------------------------------- */
/* O7: backward, push style in reverse canonical order.          */
/* State adjoints per pin/rf: mbar = dL/dmu, sbar = dL/dsigma.                */
/* Merge (Eq 4/6): A_i = LSE(A_c), w_c = exp((A_c - M)/tau) / sum (Eq 6);     */
/* hard mode is w = one-hot(c*).  With mu_i = A_i - Ns*sig_{c*} and           */
/* sig_i = sig_{c*}:                                                          */
/*   Abar_c   = w_c * mbar_i                                                  */
/*   mbar_c   = Abar_c                                                        */
/*   sbar_c   = Ns*Abar_c + [c = c*]*(sbar_i - Ns*mbar_i)                     */
/* Candidate (Eq 1-2): mbar_j[s] += mbar_c, dmean_e[rf] += mbar_c,            */
/*   sbar_j[s] += sbar_c*sig_j[s]/sig_c, dsigma_e[rf] += sbar_c*sig_e/sig_c   */
/*   (0/0 := 0).                                                              */
/* ------------------------------------------------------------------------- */
#ifdef _OPENMP
#define ORC_PUSH(x, v) do { double v_ = (v); _Pragma("omp atomic") (x) += v_; } while (0)
#else
#define ORC_PUSH(x, v) ((x) += (v))
#endif
static void backward_pin(const orc_graph* g, const topo_t* t, int32_t k, double n_sigma, double tau,
                         const double* mu, const double* sig, double* mbar, double* sbar, double* dm, double* ds,
                         cand_t* c, double* w) {
  int32_t i = t->order[k];
  if (t->fanin_ptr[k] == t->fanin_ptr[k + 1]) return;
  for (int rf = 0; rf < 2; ++rf) {
    double mb = mbar[2 * (int64_t)i + rf], sb = sbar[2 * (int64_t)i + rf];
    if (mb == 0.0 && sb == 0.0) continue;
    int n = candidates(g, t, k, rf, n_sigma, mu, sig, c);
    int b = first_argmax(c, n);
    if (tau == 0.0) {
      for (int a = 0; a < n; ++a) w[a] = (a == b) ? 1.0 : 0.0;
    } else {
      double M = c[b].A, sum = 0.0;
      for (int a = 0; a < n; ++a) sum += exp((c[a].A - M) / tau);
      for (int a = 0; a < n; ++a) w[a] = exp((c[a].A - M) / tau) / sum;   /* Eq 6 */
    }
    for (int a = 0; a < n; ++a) {
      double Abar_c = w[a] * mb;
      double mbar_c = Abar_c;
      double sbar_c = n_sigma * Abar_c + ((a == b) ? (sb - n_sigma * mb) : 0.0);
      int64_t e = c[a].arc;
      int32_t j = c[a].src;
      int s = c[a].s;
      double sig_j = sig[2 * (int64_t)j + s];
      double sig_e = g->arc_sigma[2 * e + rf];
      ORC_PUSH(mbar[2 * (int64_t)j + s], mbar_c);
      dm[2 * e + rf] += mbar_c;   /* arc e has one sink: written by this pin only */
      if (c[a].sig > 0.0) {
        ORC_PUSH(sbar[2 * (int64_t)j + s], sbar_c * sig_j / c[a].sig);
        ds[2 * e + rf] += sbar_c * sig_e / c[a].sig;
      }
    }
  }
}

int orc_backward(const orc_graph* g, double n_sigma, double tau,
                 const double* dslack, double* d_mean, double* d_sigma,
                 double* d_src_mean, double* d_src_sigma, double* abar) {
  int st = orc_validate(g, n_sigma, tau);
  if (st) return st;
  topo_t t;
  st = topo_build(g->num_pins, g->num_arcs, g->arc_from, g->arc_to, &t);
  if (st) return st;
  int32_t N = g->num_pins;
  int64_t E = g->num_arcs;
  size_t n2 = 2 * (size_t)N + 2;
  double* mu = malloc(n2 * sizeof(double));
  double* sig = malloc(n2 * sizeof(double));
  propagate(g, &t, n_sigma, tau, mu, sig, NULL, NULL, NULL);

  double* mbar = calloc(n2, sizeof(double));
  double* sbar = calloc(n2, sizeof(double));
  double* dm = calloc(2 * (size_t)E + 2, sizeof(double));
  double* ds = calloc(2 * (size_t)E + 2, sizeof(double));

  /* seeds: slack = RAT - (mu + Ns*sig) at rf*, so dL/dmu = -dslack, dL/dsig = -Ns*dslack */
  for (int32_t k = 0; k < g->num_endpoints; ++k) {
    int32_t p = g->ep_pin[k];
    double sr = g->ep_rat[2 * k + RISE] - (mu[2 * (int64_t)p + RISE] + n_sigma * sig[2 * (int64_t)p + RISE]);
    double sf = g->ep_rat[2 * k + FALL] - (mu[2 * (int64_t)p + FALL] + n_sigma * sig[2 * (int64_t)p + FALL]);
    int r = (sf < sr) ? FALL : RISE;
    double s = (r == FALL) ? sf : sr;
    double seed = dslack ? dslack[k] : (s < 0 ? 1.0 : 0.0);
    mbar[2 * (int64_t)p + r] += -seed;
    sbar[2 * (int64_t)p + r] += -n_sigma * seed;
  }

#ifdef _OPENMP
  /* all-core build: the pins of a level in parallel, pushes as atomic adds (the
   * summation order of a source's adjoint varies: equal to rounding) */
  for (int32_t l = t.num_levels - 1; l >= 0; --l) {
#pragma omp parallel
    {
      cand_t* c = malloc(sizeof(cand_t) * 2 * (size_t)max_fanin(&t));
      double* w = malloc(sizeof(double) * 2 * (size_t)max_fanin(&t));
#pragma omp for schedule(static)
      for (int32_t k = t.level_ptr[l]; k < t.level_ptr[l + 1]; ++k)
        backward_pin(g, &t, k, n_sigma, tau, mu, sig, mbar, sbar, dm, ds, c, w);
      free(c); free(w);
    }
  }
#else
  cand_t* c = malloc(sizeof(cand_t) * 2 * (size_t)max_fanin(&t));
  double* w = malloc(sizeof(double) * 2 * (size_t)max_fanin(&t));
  for (int32_t k = N - 1; k >= 0; --k) backward_pin(g, &t, k, n_sigma, tau, mu, sig, mbar, sbar, dm, ds, c, w);
  free(c); free(w);
#endif

  if (d_mean) memcpy(d_mean, dm, sizeof(double) * 2 * (size_t)E);
  if (d_sigma) memcpy(d_sigma, ds, sizeof(double) * 2 * (size_t)E);
  for (int32_t p = 0; p < N; ++p) {
    int is_src = (t.fanin_ptr[t.pos[p]] == t.fanin_ptr[t.pos[p] + 1]);
    for (int rf = 0; rf < 2; ++rf) {
      if (d_src_mean) d_src_mean[2 * (int64_t)p + rf] = is_src ? mbar[2 * (int64_t)p + rf] : 0.0;
      if (d_src_sigma) d_src_sigma[2 * (int64_t)p + rf] = is_src ? sbar[2 * (int64_t)p + rf] : 0.0;
      if (abar) abar[2 * (int64_t)p + rf] = mbar[2 * (int64_t)p + rf];
    }
  }
  free(mu); free(sig); free(mbar); free(sbar); free(dm); free(ds);
  topo_free(&t);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* Test support: near-tie taint (hard mode).  Not part of the method.         */
/* ------------------------------------------------------------------------- */
int orc_tie_taint(const orc_graph* g, double n_sigma, double eps, double margin,
                  uint8_t* fwd_taint, uint8_t* arc_taint) {
  int st = orc_validate(g, n_sigma, 0.0);
  if (st) return st;
  topo_t t;
  st = topo_build(g->num_pins, g->num_arcs, g->arc_from, g->arc_to, &t);
  if (st) return st;
  int32_t N = g->num_pins;
  int64_t E = g->num_arcs;
  size_t n2 = 2 * (size_t)N + 2;
  double* mu = malloc(n2 * sizeof(double));
  double* sig = malloc(n2 * sizeof(double));
  propagate(g, &t, n_sigma, 0.0, mu, sig, NULL, NULL, NULL);
  uint8_t* ft = calloc(n2, 1);
  uint8_t* bt = calloc(n2, 1);     /* backward: adjoint of (pin, rf) uncertain */
  uint8_t* at = calloc(2 * (size_t)E + 2, 1);
  cand_t* c = malloc(sizeof(cand_t) * 2 * (size_t)max_fanin(&t));

  /* forward taint: near tie at the merge, or a near-max candidate from a tainted source */
  for (int32_t k = 0; k < N; ++k) {
    int32_t i = t.order[k];
    if (t.fanin_ptr[k] == t.fanin_ptr[k + 1]) continue;
    for (int rf = 0; rf < 2; ++rf) {
      int n = candidates(g, &t, k, rf, n_sigma, mu, sig, c);
      int b = first_argmax(c, n);
      uint8_t x = 0;
      for (int a = 0; a < n; ++a) {
        if (a != b && c[b].A - c[a].A <= eps) x = 1;
        if (c[b].A - c[a].A <= margin && ft[2 * (int64_t)c[a].src + c[a].s]) x = 1;
      }
      ft[2 * (int64_t)i + rf] = x;
    }
  }
  /* backward taint originates at endpoints whose seed (slack sign, rf*) is
   * ambiguous: within eps of a kink, or within `margin` of one when the
   * endpoint's state is tainted (a near tie upstream moves its arrival by less
   * than margin).  A tainted endpoint whose seed is certain routes no uncertain
   * adjoint: no taint (T2). */
  for (int32_t k = 0; k < g->num_endpoints; ++k) {
    int32_t p = g->ep_pin[k];
    double ar = mu[2 * (int64_t)p] + n_sigma * sig[2 * (int64_t)p];
    double af = mu[2 * (int64_t)p + 1] + n_sigma * sig[2 * (int64_t)p + 1];
    double sr = g->ep_rat[2 * k] - ar, sf = g->ep_rat[2 * k + 1] - af;
    double s = sf < sr ? sf : sr;
    double tol = (ft[2 * (int64_t)p] || ft[2 * (int64_t)p + 1]) ? margin : eps;
    if (fabs(sr - sf) <= tol || fabs(s) <= tol) {
      bt[2 * (int64_t)p] = bt[2 * (int64_t)p + 1] = 1;
    }
  }
  /* reverse: where the oracle (or an uncertain upstream) routes adjoint, an
   * ambiguous merge taints every candidate within `margin` of the max, and an
   * unambiguous merge with an uncertain adjoint taints only its winner. */
  double* mb = malloc(n2 * sizeof(double));
  orc_backward(g, n_sigma, 0.0, NULL, NULL, NULL, NULL, NULL, mb);
  for (int32_t k = N - 1; k >= 0; --k) {
    int32_t i = t.order[k];
    if (t.fanin_ptr[k] == t.fanin_ptr[k + 1]) continue;
    for (int rf = 0; rf < 2; ++rf) {
      int64_t q = 2 * (int64_t)i + rf;
      if (!(bt[q] || mb[q] != 0.0)) continue;
      int n = candidates(g, &t, k, rf, n_sigma, mu, sig, c);
      int b = first_argmax(c, n);
      int amb = ft[q];
      for (int a = 0; a < n; ++a) if (a != b && c[b].A - c[a].A <= eps) amb = 1;
      for (int a = 0; a < n; ++a) {
        int hit = amb ? (c[b].A - c[a].A <= margin) : (bt[q] && a == b);
        if (hit) {
          bt[2 * (int64_t)c[a].src + c[a].s] = 1;
          at[2 * (int64_t)c[a].arc + rf] = 1;
        }
      }
    }
  }
  free(mb);
  if (fwd_taint) memcpy(fwd_taint, ft, 2 * (size_t)N);
  if (arc_taint) memcpy(arc_taint, at, 2 * (size_t)E);
  free(c); free(ft); free(bt); free(at); free(mu); free(sig);
  topo_free(&t);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* NEXT 1: Top-K statistical arrival propagation with unique   */
/* startpoints (Alg 1 + Alg 2) and CPPR-aware slack         */
/* (endpoint required times "associated with respective startpoints").*/
/*                                                                           */
/* Per pin and sink transition rf a queue of K entries {A, mu, sig, SP},      */
/* descending in A; an empty entry has A = -inf and SP = -1 (reading R13).    */
/* Startpoints: entry 0 = the clock arrival distribution with SP = the pin    */
/* itself (caller id).  Other pins, Alg 1 l.7: for k = 0..K-1 (outer), for    */
/* each fanin arc in row order (inner), for s in S(rf, u) (reading R3), the   */
/* parent's entry k of transition s -- if it exists -- gives a candidate      */
/* (Eq 1-3, l.9-16) that is offered to the queue by Alg 2 (l.17).             */
/* ------------------------------------------------------------------------- */
typedef struct { double A, mu, sig; int32_t sp; } tk_ent;

/* Alg 2: in-place update of one queue (q[0..K-1], descending in A). */
static void alg2_update(tk_ent* q, int K, tk_ent nw) {
  /* Step 1 (l.2-8): is SP_new already in the queue? */
  for (int j = 0; j < K; ++j) {
    if (q[j].sp == nw.sp) {
      if (nw.A > q[j].A) {                       /* l.4: replace only if strictly greater */
        q[j] = nw;                               /* l.5-6 */
        /* reading R13: the in-place update can break descending order;
         * re-bubble the entry up past strictly smaller entries */
        while (j > 0 && q[j].A > q[j - 1].A) { tk_ent x = q[j]; q[j] = q[j - 1]; q[j - 1] = x; --j; }
      }
      return;                                    /* l.8: exit once SP_new is found */
    }
  }
  /* Step 2 (l.9-): SP_new not found -- insert before the first smaller entry,
   * shifting the rest down; the last entry falls off ("checks whether
   * A_new exceeds the smallest arrival time ... inserted in the appropriate
   * position to maintain descending order") */
  for (int j = 0; j < K; ++j) {
    if (nw.A > q[j].A) {
      for (int m = K - 1; m > j; --m) q[m] = q[m - 1];
      q[j] = nw;
      return;
    }
  }
}

int orc_topk_forward(const orc_graph* g, double n_sigma, int32_t K, double* A, double* mu,
                     double* sig, int32_t* sp) {
  int st = orc_validate(g, n_sigma, 0.0);
  if (st) return st;
  if (K < 1) return 1;
  topo_t t;
  st = topo_build(g->num_pins, g->num_arcs, g->arc_from, g->arc_to, &t);
  if (st) return st;
  int32_t N = g->num_pins;
  tk_ent* Q = malloc(sizeof(tk_ent) * ((size_t)N * 2 * K + 1));  /* [N][2][K], caller-indexed */
  const tk_ent empty = {-INFINITY, 0.0, 0.0, -1};
  for (int32_t k = 0; k < N; ++k) {
    int32_t i = t.order[k];
    for (int rf = 0; rf < 2; ++rf) {
      tk_ent* q = Q + ((size_t)i * 2 + rf) * K;
      for (int m = 0; m < K; ++m) q[m] = empty;
      if (t.fanin_ptr[k] == t.fanin_ptr[k + 1]) {
        /* startpoint: clock arrival, corner via Eq 3; SP = this pin */
        q[0].mu = g->src_mean ? g->src_mean[2 * (int64_t)i + rf] : 0.0;
        q[0].sig = g->src_sigma ? g->src_sigma[2 * (int64_t)i + rf] : 0.0;
        q[0].A = q[0].mu + n_sigma * q[0].sig;
        q[0].sp = i;
        continue;
      }
      for (int kk = 0; kk < K; ++kk) {                              /* Alg 1 l.7: k outer */
        for (int32_t r = t.fanin_ptr[k]; r < t.fanin_ptr[k + 1]; ++r) { /* parents, row order */
          int32_t e = t.fanin_arc[r];
          int32_t j = g->arc_from[e];
          int ss[2];
          int ns = sources_of(rf, g->arc_unate[e], ss);             /* Alg 1 l.8, reading R3 */
          for (int a = 0; a < ns; ++a) {
            const tk_ent* p = Q + ((size_t)j * 2 + ss[a]) * K + kk;
            if (p->sp < 0) continue;                                /* no k-th arrival at the parent */
            double arc_mean = g->arc_mean[2 * (int64_t)e + rf];
            double arc_std = g->arc_sigma[2 * (int64_t)e + rf];
            tk_ent c;
            c.mu = p->mu + arc_mean;                                /* l.12, Eq 1 */
            c.sig = sqrt(p->sig * p->sig + arc_std * arc_std);      /* l.13, Eq 2 */
            c.A = c.mu + n_sigma * c.sig;                           /* l.14, Eq 3 */
            c.sp = p->sp;                                           /* l.16 */
            alg2_update(q, K, c);                                   /* l.17 */
          }
        }
      }
    }
  }
  for (size_t x = 0; x < (size_t)N * 2 * K; ++x) {
    if (A) A[x] = Q[x].A;
    if (mu) mu[x] = Q[x].mu;
    if (sig) sig[x] = Q[x].sig;
    if (sp) sp[x] = Q[x].sp;
  }
  free(Q);
  topo_free(&t);
  return 0;
}

/* CPPR slack: endpoint required times are associated with
 * startpoints.  rat_ptr[P+1] / rat_sp[] / rat_val[][2]: per endpoint, a list of
 * (startpoint caller id, RAT{R,F}); a startpoint not in its endpoint's list
 * takes the endpoint's default ep_rat.  slack = min over rf (R first) and over
 * the K queue entries (in queue order) of RAT(ep, SP_k)[rf] - A_k[rf]; the
 * first minimum wins ties.  WNS / TNS / violations as in orc_slack.
 * Outputs: slack[P], rf_star[P], k_star[P], sp_star[P] (caller id). */
int orc_topk_slack(const orc_graph* g, int32_t K, const double* A, const int32_t* sp,
                   const int32_t* rat_ptr, const int32_t* rat_sp, const double* rat_val,
                   double* slack, uint8_t* rf_star, int32_t* k_star, int32_t* sp_star,
                   double* wns, double* tns, int32_t* num_viol) {
  double w = 0.0, tt = 0.0;
  int32_t nv = 0;
  for (int32_t e = 0; e < g->num_endpoints; ++e) {
    int32_t p = g->ep_pin[e];
    double best = INFINITY;
    int br = 0, bk = 0;
    int32_t bsp = -1;
    for (int rf = 0; rf < 2; ++rf) {
      for (int k = 0; k < K; ++k) {
        size_t x = ((size_t)p * 2 + rf) * K + k;
        if (sp[x] < 0) continue;
        double rat = g->ep_rat[2 * e + rf];
        if (rat_ptr)
          for (int32_t m = rat_ptr[e]; m < rat_ptr[e + 1]; ++m)
            if (rat_sp[m] == sp[x]) { rat = rat_val[2 * (int64_t)m + rf]; break; }
        double s = rat - A[x];
        if (s < best) { best = s; br = rf; bk = k; bsp = sp[x]; }
      }
    }
    if (slack) slack[e] = best;
    if (rf_star) rf_star[e] = (uint8_t)br;
    if (k_star) k_star[e] = bk;
    if (sp_star) sp_star[e] = bsp;
    if (best < 0) { tt += best; ++nv; }
    if (best < w) w = best;
  }
  if (wns) *wns = w;
  if (tns) *tns = tt;
  if (num_viol) *num_viol = nv;
  return 0;
}

/* Test support (T9): which Top-K queue rows may legitimately hold a
 * different startpoint SET on another correct implementation.  By Alg 2
 * a queue ends as the K largest per-startpoint maxima of its candidates, so its
 * set is ambiguous only where (a) the K-th and (K+1)-th per-startpoint maxima are
 * within eps (a near tie at the eviction boundary), or (b) a parent row's set is
 * ambiguous and one of its uncertain entries could reach this queue.  A tainted
 * row carries hi = an upper bound on the arrival of any entry whose membership is
 * uncertain; through arc e an uncertain parent entry A = mu + n sigma moves to
 * A' = A + mean_e + n (sqrt(sigma^2 + std_e^2) - sigma) <= A + mean_e + n std_e
 * (Eq 1-3), so it can enter a full queue only if hi_p + mean_e + n std_e reaches
 * the K-th kept arrival minus eps; a queue that is not full takes any candidate.
 * Output: taint[N][2] (caller ids).  Order ties inside a row (two kept entries
 * within eps) are not flagged here: they reorder, not change, the set. */
typedef struct { double A; int32_t sp; } tk_cand;
static int cmp_cand_sp(const void* a, const void* b) {
  const tk_cand *x = a, *y = b;
  if (x->sp != y->sp) return x->sp < y->sp ? -1 : 1;
  return (x->A > y->A) ? -1 : (x->A < y->A);
}
static int cmp_cand_desc(const void* a, const void* b) {
  const tk_cand *x = a, *y = b;
  return (x->A > y->A) ? -1 : (x->A < y->A);
}

int orc_topk_taint(const orc_graph* g, double n_sigma, int32_t K, double eps, uint8_t* taint) {
  int st = orc_validate(g, n_sigma, 0.0);
  if (st) return st;
  if (K < 1) return 1;
  int32_t N = g->num_pins;
  size_t nq = (size_t)N * 2 * K;
  double* mu = malloc(sizeof(double) * (nq + 1));
  double* sig = malloc(sizeof(double) * (nq + 1));
  int32_t* sp = malloc(sizeof(int32_t) * (nq + 1));
  st = orc_topk_forward(g, n_sigma, K, NULL, mu, sig, sp);
  if (st) { free(mu); free(sig); free(sp); return st; }
  topo_t t;
  st = topo_build(g->num_pins, g->num_arcs, g->arc_from, g->arc_to, &t);
  if (st) { free(mu); free(sig); free(sp); return st; }
  uint8_t* tn = calloc(2 * (size_t)N + 2, 1);
  double* hi = malloc(sizeof(double) * (2 * (size_t)N + 2));
  int32_t maxfi = max_fanin(&t);
  tk_cand* c = malloc(sizeof(tk_cand) * ((size_t)maxfi * 2 * K + 1));
  for (int32_t k = 0; k < N; ++k) {
    int32_t i = t.order[k];
    if (t.fanin_ptr[k] == t.fanin_ptr[k + 1]) continue;        /* startpoint: one certain entry */
    for (int rf = 0; rf < 2; ++rf) {
      int n = 0;
      double U = -INFINITY;                                      /* bound on uncertain candidates */
      int any_parent = 0;
      for (int32_t r = t.fanin_ptr[k]; r < t.fanin_ptr[k + 1]; ++r) {
        int32_t e = t.fanin_arc[r];
        int32_t j = g->arc_from[e];
        int ss[2];
        int ns = sources_of(rf, g->arc_unate[e], ss);
        double am = g->arc_mean[2 * (int64_t)e + rf], as = g->arc_sigma[2 * (int64_t)e + rf];
        for (int a = 0; a < ns; ++a) {
          size_t row = (size_t)j * 2 + ss[a];
          for (int m = 0; m < K; ++m) {
            size_t x = row * K + m;
            if (sp[x] < 0) continue;
            c[n].A = mu[x] + am + n_sigma * sqrt(sig[x] * sig[x] + as * as);   /* Eq 1-3 */
            c[n].sp = sp[x];
            ++n;
          }
          if (tn[row]) {
            any_parent = 1;
            double u = hi[row] + am + n_sigma * as;
            if (u > U) U = u;
          }
        }
      }
      /* per-startpoint maxima, descending */
      qsort(c, (size_t)n, sizeof(tk_cand), cmp_cand_sp);
      int nu = 0;
      for (int a = 0; a < n; ++a)
        if (a == 0 || c[a].sp != c[a - 1].sp) c[nu++] = c[a];
      qsort(c, (size_t)nu, sizeof(tk_cand), cmp_cand_desc);
      int64_t q = 2 * (int64_t)i + rf;
      double h = -INFINITY;
      int x = 0;
      if (nu > K && c[K - 1].A - c[K].A <= eps) { x = 1; h = c[K - 1].A + eps; }     /* (a) */
      if (any_parent && (nu < K || U >= c[K - 1].A - eps)) {                        /* (b) */
        x = 1;
        double b = (nu >= K && c[K - 1].A + eps > U) ? c[K - 1].A + eps : U + eps;
        if (b > h) h = b;
      }
      tn[q] = (uint8_t)x;
      hi[q] = h;
    }
  }
  if (taint) memcpy(taint, tn, 2 * (size_t)N);
  free(c); free(hi); free(tn); free(mu); free(sig); free(sp);
  topo_free(&t);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* NEXT 2: Clark moment-matching statistical max, the merge    */
/* the north star names beside the paper's smooth max.  The state of a pin is */
/* the Gaussian (mu, V = sigma^2) per rf; a candidate is (mu_j[s] + mean_e,   */
/* V_j[s] + std_e^2) (Eq 1-2); the merge folds the candidates in canonical    */
/* order (fanin row, then s = rf before ~rf) with Clark's two-input max of    */
/* independent Gaussians (reading R20: rho = 0):                              */
/*   a = sqrt(V1 + V2), alpha = (mu1 - mu2) / a                               */
/*   mu  = mu1 Phi(alpha) + mu2 Phi(-alpha) + a phi(alpha)                    */
/*   E2  = (mu1^2 + V1) Phi(alpha) + (mu2^2 + V2) Phi(-alpha)                 */
/*         + (mu1 + mu2) a phi(alpha),      V = E2 - mu^2                     */
/* (a = 0: the hard max, first input wins ties).  Endpoint arrival Eq 3:      */
/* A = mu + N_sigma sqrt(V); slack / WNS / TNS as O6.                         */
/* ------------------------------------------------------------------------- */
static double Phi_(double x) { return 0.5 * erfc(-x / sqrt(2.0)); }
static double phi_(double x) { return exp(-0.5 * x * x) / sqrt(2.0 * 3.14159265358979323846); }

static void clark2(double m1, double v1, double m2, double v2, double* m, double* v) {
  double a2 = v1 + v2;
  if (!(a2 > 0.0)) {                     /* both deterministic: hard max, first wins ties */
    if (m2 > m1) { *m = m2; *v = v2; } else { *m = m1; *v = v1; }
    return;
  }
  double a = sqrt(a2), al = (m1 - m2) / a;
  double P = Phi_(al), Q = Phi_(-al), p = phi_(al);
  *m = m1 * P + m2 * Q + a * p;
  double e2 = (m1 * m1 + v1) * P + (m2 * m2 + v2) * Q + (m1 + m2) * a * p;
  *v = e2 - (*m) * (*m);
  if (*v < 0.0) *v = 0.0;
}

/* Jacobian of clark2: d(mu, V)/d(m1, v1, m2, v2), rows J[0] = dmu, J[1] = dV */
static void clark2_jac(double m1, double v1, double m2, double v2, double J[2][4]) {
  double a2 = v1 + v2;
  if (!(a2 > 0.0)) {
    int second = m2 > m1;
    for (int r = 0; r < 2; ++r) for (int c = 0; c < 4; ++c) J[r][c] = 0.0;
    J[0][second ? 2 : 0] = 1.0;
    J[1][second ? 3 : 1] = 1.0;
    return;
  }
  double a = sqrt(a2), al = (m1 - m2) / a;
  double P = Phi_(al), Q = Phi_(-al), p = phi_(al);
  double mu = m1 * P + m2 * Q + a * p;
  /* d mu */
  double dm1 = P, dm2 = Q, dv = p / (2.0 * a);
  /* d E2 (derived from the closed form; pinned by finite differences in tests) */
  double e_m1 = 2.0 * m1 * P + a * p + (p / a) * (v1 - v2);
  double e_m2 = 2.0 * m2 * Q + a * p - (p / a) * (v1 - v2);
  double e_a = (m1 + m2) * p - al * p * (v1 - v2) / a;
  double e_v1 = P + e_a / (2.0 * a), e_v2 = Q + e_a / (2.0 * a);
  J[0][0] = dm1; J[0][1] = dv; J[0][2] = dm2; J[0][3] = dv;
  J[1][0] = e_m1 - 2.0 * mu * dm1;
  J[1][1] = e_v1 - 2.0 * mu * dv;
  J[1][2] = e_m2 - 2.0 * mu * dm2;
  J[1][3] = e_v2 - 2.0 * mu * dv;
}

typedef struct { int32_t arc, src; int s; double mu, v; } ccand_t;

static int clark_candidates(const orc_graph* g, const topo_t* t, int32_t k, int rf, const double* M,
                            const double* V, ccand_t* c) {
  int n = 0;
  for (int32_t q = t->fanin_ptr[k]; q < t->fanin_ptr[k + 1]; ++q) {
    int32_t e = t->fanin_arc[q], j = g->arc_from[e];
    int ss[2];
    int ns = sources_of(rf, g->arc_unate[e], ss);
    for (int a = 0; a < ns; ++a) {
      double sd = g->arc_sigma[2 * (int64_t)e + rf];
      c[n].arc = e; c[n].src = j; c[n].s = ss[a];
      c[n].mu = M[2 * (int64_t)j + ss[a]] + g->arc_mean[2 * (int64_t)e + rf];   /* Eq 1 */
      c[n].v = V[2 * (int64_t)j + ss[a]] + sd * sd;                              /* Eq 2 */
      ++n;
    }
  }
  return n;
}

static void clark_propagate(const orc_graph* g, const topo_t* t, double* M, double* V) {
  ccand_t* c = malloc(sizeof(ccand_t) * 2 * (size_t)max_fanin(t));
  for (int32_t k = 0; k < t->n; ++k) {
    int32_t i = t->order[k];
    for (int rf = 0; rf < 2; ++rf) {
      int64_t x = 2 * (int64_t)i + rf;
      if (t->fanin_ptr[k] == t->fanin_ptr[k + 1]) {     /* startpoint */
        double s = g->src_sigma ? g->src_sigma[x] : 0.0;
        M[x] = g->src_mean ? g->src_mean[x] : 0.0;
        V[x] = s * s;
        continue;
      }
      int n = clark_candidates(g, t, k, rf, M, V, c);
      double m = c[0].mu, v = c[0].v;
      for (int a = 1; a < n; ++a) clark2(m, v, c[a].mu, c[a].v, &m, &v);   /* fold in order */
      M[x] = m;
      V[x] = v;
    }
  }
  free(c);
}

int orc_clark_forward(const orc_graph* g, double n_sigma, double* A, double* mu, double* sig) {
  int st = orc_validate(g, n_sigma, 0.0);
  if (st) return st;
  topo_t t;
  st = topo_build(g->num_pins, g->num_arcs, g->arc_from, g->arc_to, &t);
  if (st) return st;
  size_t n2 = 2 * (size_t)g->num_pins + 2;
  double* M = malloc(n2 * sizeof(double));
  double* V = malloc(n2 * sizeof(double));
  clark_propagate(g, &t, M, V);
  for (int64_t x = 0; x < 2 * (int64_t)g->num_pins; ++x) {
    if (A) A[x] = M[x] + n_sigma * sqrt(V[x]);   /* Eq 3 */
    if (mu) mu[x] = M[x];
    if (sig) sig[x] = sqrt(V[x]);
  }
  free(M); free(V);
  topo_free(&t);
  return 0;
}

/* Backward of the Clark path (push style, reverse canonical order).  Seeds:
 * slack = RAT - (mu + Ns sqrt(V)) at rf*, so dL/dmu = -seed and
 * dL/dV = -seed Ns / (2 sqrt(V)) (0 if V = 0).  Through the fold: reverse
 * over the prefix results r_k = clark(r_{k-1}, c_k) with clark2_jac.  A
 * candidate passes its adjoint to the source (mu, V) and to the arc:
 * d mean_e += mubar_c, d sigma_e += 2 std_e Vbar_c; sources: d src_mean =
 * mubar, d src_sigma = 2 sigma_src Vbar. */
int orc_clark_backward(const orc_graph* g, double n_sigma, const double* dslack, double* d_mean,
                       double* d_sigma, double* d_src_mean, double* d_src_sigma) {
  int st = orc_validate(g, n_sigma, 0.0);
  if (st) return st;
  topo_t t;
  st = topo_build(g->num_pins, g->num_arcs, g->arc_from, g->arc_to, &t);
  if (st) return st;
  int32_t N = g->num_pins;
  int64_t E = g->num_arcs;
  size_t n2 = 2 * (size_t)N + 2;
  double* M = malloc(n2 * sizeof(double));
  double* V = malloc(n2 * sizeof(double));
  clark_propagate(g, &t, M, V);
  double* mb = calloc(n2, sizeof(double));
  double* vb = calloc(n2, sizeof(double));
  double* dm = calloc(2 * (size_t)E + 2, sizeof(double));
  double* ds = calloc(2 * (size_t)E + 2, sizeof(double));
  for (int32_t k = 0; k < g->num_endpoints; ++k) {
    int32_t p = g->ep_pin[k];
    double ar = M[2 * (int64_t)p] + n_sigma * sqrt(V[2 * (int64_t)p]);
    double af = M[2 * (int64_t)p + 1] + n_sigma * sqrt(V[2 * (int64_t)p + 1]);
    double sr = g->ep_rat[2 * k] - ar, sf = g->ep_rat[2 * k + 1] - af;
    int r = (sf < sr) ? FALL : RISE;
    double s = (r == FALL) ? sf : sr;
    double seed = dslack ? dslack[k] : (s < 0 ? 1.0 : 0.0);
    int64_t x = 2 * (int64_t)p + r;
    mb[x] += -seed;
    if (V[x] > 0.0) vb[x] += -seed * n_sigma / (2.0 * sqrt(V[x]));
  }
  int mf = 2 * max_fanin(&t);
  ccand_t* c = malloc(sizeof(ccand_t) * (size_t)mf);
  double* rm = malloc(sizeof(double) * (size_t)mf);
  double* rv = malloc(sizeof(double) * (size_t)mf);
  double* cmb = malloc(sizeof(double) * (size_t)mf);
  double* cvb = malloc(sizeof(double) * (size_t)mf);
  for (int32_t k = N - 1; k >= 0; --k) {
    int32_t i = t.order[k];
    if (t.fanin_ptr[k] == t.fanin_ptr[k + 1]) continue;
    for (int rf = 0; rf < 2; ++rf) {
      int64_t x = 2 * (int64_t)i + rf;
      if (mb[x] == 0.0 && vb[x] == 0.0) continue;
      int n = clark_candidates(g, &t, k, rf, M, V, c);
      rm[0] = c[0].mu; rv[0] = c[0].v;                 /* prefix results of the fold */
      for (int a = 1; a < n; ++a) clark2(rm[a - 1], rv[a - 1], c[a].mu, c[a].v, &rm[a], &rv[a]);
      double um = mb[x], uv = vb[x];                   /* adjoint of r_{n-1} */
      for (int a = n - 1; a >= 1; --a) {
        double J[2][4];
        clark2_jac(rm[a - 1], rv[a - 1], c[a].mu, c[a].v, J);
        cmb[a] = um * J[0][2] + uv * J[1][2];
        cvb[a] = um * J[0][3] + uv * J[1][3];
        double pm = um * J[0][0] + uv * J[1][0];
        double pv = um * J[0][1] + uv * J[1][1];
        um = pm; uv = pv;
      }
      cmb[0] = um; cvb[0] = uv;
      for (int a = 0; a < n; ++a) {
        int64_t e = c[a].arc;
        int64_t y = 2 * (int64_t)c[a].src + c[a].s;
        mb[y] += cmb[a];
        vb[y] += cvb[a];
        dm[2 * e + rf] += cmb[a];
        ds[2 * e + rf] += 2.0 * g->arc_sigma[2 * e + rf] * cvb[a];
      }
    }
  }
  if (d_mean) memcpy(d_mean, dm, sizeof(double) * 2 * (size_t)E);
  if (d_sigma) memcpy(d_sigma, ds, sizeof(double) * 2 * (size_t)E);
  for (int32_t p = 0; p < N; ++p) {
    int is_src = (t.fanin_ptr[t.pos[p]] == t.fanin_ptr[t.pos[p] + 1]);
    for (int rf = 0; rf < 2; ++rf) {
      int64_t x = 2 * (int64_t)p + rf;
      double ssd = g->src_sigma ? g->src_sigma[x] : 0.0;
      if (d_src_mean) d_src_mean[x] = is_src ? mb[x] : 0.0;
      if (d_src_sigma) d_src_sigma[x] = is_src ? 2.0 * ssd * vb[x] : 0.0;
    }
  }
  free(c); free(rm); free(rv); free(cmb); free(cvb);
  free(M); free(V); free(mb); free(vb); free(dm); free(ds);
  topo_free(&t);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* NEXT 4: INSTA-Place timing objective, Eq 7:    */
/*   L = lambda_RC * sum_k (|x_f - x_t| + |y_f - y_t|) * w_k                  */
/* over every arc k = (f -> t) with weight w_k (reading R21: w_k = the arc's  */
/* timing sensitivity -dTNS/d(delay), zero for non-critical arcs), and its    */
/* gradient w.r.t. the pin positions (subgradient sign(0) = 0).  Positions     */
/* and weights in caller order.                                               */
/* ------------------------------------------------------------------------- */
static double sgn(double d) { return d > 0.0 ? 1.0 : (d < 0.0 ? -1.0 : 0.0); }

int orc_timing_loss(const orc_graph* g, const double* x, const double* y, const double* w, double lambda_rc,
                    double* loss, double* gx, double* gy) {
  if (!g || !x || !y || !w) return 1;
  double L = 0.0;
  if (gx) memset(gx, 0, sizeof(double) * (size_t)g->num_pins);
  if (gy) memset(gy, 0, sizeof(double) * (size_t)g->num_pins);
  for (int64_t k = 0; k < g->num_arcs; ++k) {
    int32_t f = g->arc_from[k], t = g->arc_to[k];
    double dx = x[f] - x[t], dy = y[f] - y[t];
    L += (fabs(dx) + fabs(dy)) * w[k];
    if (gx) { gx[f] += lambda_rc * w[k] * sgn(dx); gx[t] -= lambda_rc * w[k] * sgn(dx); }
    if (gy) { gy[f] += lambda_rc * w[k] * sgn(dy); gy[t] -= lambda_rc * w[k] * sgn(dy); }
  }
  if (loss) *loss = lambda_rc * L;
  return 0;
}

/* ------------------------------------------------------------------------- */
/* NEXT 3: INSTA-Size stage gradients: "the timing    */
/* gradient of each stage (i.e., the gradient sum of a cell arc and its       */
/* driving net arc)".  Reading R22: the stage of a cell arc e_c = (p -> o) is  */
/* e_c plus the single net arc into p when p has exactly one fanin arc and it  */
/* is a net arc; stage_grad[e_c] = sum_rf d_mean[e_c][rf] + sum_rf            */
/* d_mean[e_n][rf]; 0 for net arcs.  arc_class: 0 net, 1 cell (caller order). */
/* ------------------------------------------------------------------------- */
int orc_stage_gradients(const orc_graph* g, const uint8_t* arc_class, const double* d_mean, double* out) {
  if (!g || !arc_class || !d_mean || !out) return 1;
  int32_t N = g->num_pins;
  int32_t* nin = calloc((size_t)N + 1, sizeof(int32_t));
  int64_t* in_arc = malloc(sizeof(int64_t) * ((size_t)N + 1));
  for (int32_t p = 0; p < N; ++p) in_arc[p] = -1;
  for (int64_t e = 0; e < g->num_arcs; ++e) { nin[g->arc_to[e]]++; in_arc[g->arc_to[e]] = e; }
  for (int64_t e = 0; e < g->num_arcs; ++e) {
    if (arc_class[e] != 1) { out[e] = 0.0; continue; }
    double s = d_mean[2 * e] + d_mean[2 * e + 1];
    int32_t p = g->arc_from[e];
    if (nin[p] == 1 && arc_class[in_arc[p]] == 0) s += d_mean[2 * in_arc[p]] + d_mean[2 * in_arc[p] + 1];
    out[e] = s;
  }
  free(nin); free(in_arc);
  return 0;
}
