/*
 * oracle.h -- plain, slow, fp64 CPU oracle of INSTA's K=1 hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load liboracle.so.  It
 * shares no code, header, table or constant with the CUDA path
 * (paper_conf_dac_lugklr25_b200/csrc); neither includes the other.
 *
 * Every function follows PAPER.md (cited as P:Lnn) step by step, in the
 * readings listed in DESIGN.md §3.  All arrays are in CALLER order (the ids the
 * user passed); the oracle levelizes on its own (Kahn).
 *
 * Status codes: 0 ok, 1 bad argument, 2 combinational cycle.
 */
#ifndef INSTA_ORACLE_H
#define INSTA_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int32_t num_pins;
  int64_t num_arcs;
  const int32_t* arc_from;   /* [E] */
  const int32_t* arc_to;     /* [E] */
  const uint8_t* arc_unate;  /* [E] 0 POS, 1 NEG, 2 NON */
  const double* arc_mean;    /* [E][2] {R,F}, indexed by the SINK transition (Alg 1 l.12) */
  const double* arc_sigma;   /* [E][2] */
  const double* src_mean;    /* [N][2] or NULL (=0); used at indeg-0 pins */
  const double* src_sigma;   /* [N][2] or NULL (=0) */
  int32_t num_endpoints;
  const int32_t* ep_pin;     /* [P] */
  const double* ep_rat;      /* [P][2] */
} orc_graph;

/* O2: Kahn levelization.  level[N] caller-indexed; order[N] = caller pin
 * at each canonical position (sorted by (level, pin id)); fanin_ptr/fanout_ptr
 * [N+1] over canonical positions; fanin_arc/fanout_arc [E] caller arc ids,
 * ascending within a row.  Any output may be NULL. */
int orc_levelize(int32_t num_pins, int64_t num_arcs, const int32_t* arc_from,
                 const int32_t* arc_to, int32_t* level, int32_t* order,
                 int32_t* fanin_ptr, int32_t* fanin_arc, int32_t* fanout_ptr,
                 int32_t* fanout_arc, int32_t* num_levels);

/* O1 validation of a graph + options. */
int orc_validate(const orc_graph* g, double n_sigma, double tau);

/* O3-O5 forward.  A[N][2] corner arrival, sig[N][2] sigma, mu[N][2] = A - Nsig*sig.
 * win_arc[N][2]/win_s[N][2]: the first arg-max candidate (arc id, source rf),
 * -1 at sources.  gap[N][2]: A(best) - A(second best) (+inf if one candidate).
 * Outputs other than A may be NULL. */
int orc_forward(const orc_graph* g, double n_sigma, double tau, double* A,
                double* sig, double* mu, int32_t* win_arc, int8_t* win_s,
                double* gap);

/* O6 slack: slack[P], rf_star[P] (0 R, 1 F; tie -> R), summary. */
int orc_slack(const orc_graph* g, const double* A, double* slack,
              uint8_t* rf_star, double* wns, double* tns, int32_t* num_viol);

/* O7 backward (push style, reverse canonical order).  dslack[P] = dL/dslack
 * per endpoint, or NULL for L = TNS (seed 1 where slack < 0).  Outputs (any
 * may be NULL): d_mean[E][2], d_sigma[E][2], d_src_mean[N][2],
 * d_src_sigma[N][2], abar[N][2] (adjoint of each pin's corner arrival). */
int orc_backward(const orc_graph* g, double n_sigma, double tau,
                 const double* dslack, double* d_mean, double* d_sigma,
                 double* d_src_mean, double* d_src_sigma, double* abar);

/* Test support (not part of the method): near-tie taint masks for fp32-vs-fp64
 * comparisons in hard mode.  fwd_taint[N][2]: the pin's state may legitimately
 * differ because a merge at or upstream of it is within `eps` of a tie
 * (propagated through candidates within `margin` of the max).  arc_taint[E][2]:
 * the arc's mu-gradient may legitimately differ (backward ambiguity). */
int orc_tie_taint(const orc_graph* g, double n_sigma, double eps, double margin,
                  uint8_t* fwd_taint, uint8_t* arc_taint);

/* NEXT 1: Top-K unique-startpoint propagation (Alg 1 + Alg 2).
 * Outputs [N][2][K] caller-indexed, each queue descending in A; empty entries
 * have A = -inf and sp = -1.  sp = caller id of the startpoint pin. */
int orc_topk_forward(const orc_graph* g, double n_sigma, int32_t K, double* A, double* mu,
                     double* sig, int32_t* sp);

/* CPPR slack over the Top-K queues: per endpoint e the list
 * rat_ptr[e]..rat_ptr[e+1] of (rat_sp, rat_val{R,F}) overrides the default
 * ep_rat for those startpoints.  rat_ptr may be NULL (no overrides). */
int orc_topk_slack(const orc_graph* g, int32_t K, const double* A, const int32_t* sp,
                   const int32_t* rat_ptr, const int32_t* rat_sp, const double* rat_val,
                   double* slack, uint8_t* rf_star, int32_t* k_star, int32_t* sp_star,
                   double* wns, double* tns, int32_t* num_viol);
/* Test support: Top-K queue rows whose startpoint set is legitimately ambiguous
 * (near tie at the eviction boundary, propagated); taint[N][2]. */
int orc_topk_taint(const orc_graph* g, double n_sigma, int32_t K, double eps, uint8_t* taint);

/* NEXT 2: Clark moment-matching merge (reading R20, rho = 0), folded in
 * candidate order.  A/mu/sig [N][2] caller-indexed (sig = sqrt(V)). */
int orc_clark_forward(const orc_graph* g, double n_sigma, double* A, double* mu, double* sig);

/* Backward of the Clark path: dL/d(arc mean), dL/d(arc sigma) [E][2],
 * dL/d(src mean / sigma) [N][2]; dslack = NULL means L = TNS.  Any output may be NULL. */
int orc_clark_backward(const orc_graph* g, double n_sigma, const double* dslack, double* d_mean,
                       double* d_sigma, double* d_src_mean, double* d_src_sigma);

/* NEXT 4: Eq 7 timing objective and its gradient w.r.t. pin x/y (caller order). */
int orc_timing_loss(const orc_graph* g, const double* x, const double* y, const double* w, double lambda_rc,
                    double* loss, double* gx, double* gy);

/* NEXT 3: INSTA-Size stage gradients (reading R22), out[E] caller order. */
int orc_stage_gradients(const orc_graph* g, const uint8_t* arc_class, const double* d_mean, double* out);

#ifdef __cplusplus
}
#endif
#endif
