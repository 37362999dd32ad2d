/*
 * insta.h -- C ABI of the B200-native INSTA hot path (libinsta.so).
 *
 * INSTA (Lu et al., DAC'25; /root/reference/PAPER.md, cited P:Lnn) propagates
 * statistical (POCV) arrival times level by level over a timing graph whose arc
 * delays are already known, ends in endpoint slack and WNS/TNS, and returns
 * timing gradients dTNS/d(arc delay) through a backward pass.  This header is
 * the boundary: plain C types, plain pointers (host or device as stated), no
 * C++ types, no exceptions.  Every entry point returns an insta_status; on a
 * non-OK status insta_last_error() returns a thread-local message.
 *
 * Conventions (all entry points)
 *  - Pin ids 0..num_pins-1 and arc ids 0..num_arcs-1 are CALLER ids; the
 *    internal level-ordered permutation is hidden except via insta_graph_export.
 *  - rf index 0 = rise (R), 1 = fall (F).  "[n][2]" arrays are row-major
 *    {R, F} pairs of float32 (ps).
 *  - Arc delays are indexed by the SINK transition (Alg 1 l.12-13); the
 *    source transition is ~rf for negative-unate arcs (Alg 1 l.8) and
 *    both transitions for non-unate arcs (reading R3).
 *  - Device pointers are caller-owned device memory on the graph's device
 *    (e.g. torch tensor data_ptr()); the library never keeps a caller pointer
 *    past the call.  All device work is enqueued on the caller's stream
 *    (cudaStream_t passed as void*; NULL = legacy default stream).  Only
 *    insta_graph_create / destroy / export / levelize synchronize implicitly;
 *    passing a non-NULL insta_summary* also synchronizes the stream.
 *  - One graph must not be used from two host threads at once.
 *  - Errors: INSTA_E_ARG (bad id, NaN/Inf, sigma < 0, duplicate endpoint,
 *    tau < 0, n_sigma < 0, NULL required pointer, size limits: num_pins < 2^29,
 *    num_arcs < 2^31), INSTA_E_CYCLE (combinational loop), INSTA_E_STATE (call
 *    out of order, e.g. backward before forward), INSTA_E_CUDA / INSTA_E_NOMEM
 *    (runtime failures; the graph is then unusable and must be destroyed).
 */
#ifndef INSTA_H
#define INSTA_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct insta_graph insta_graph; /* opaque; owns all of its device memory */

typedef enum {
  INSTA_OK = 0,
  INSTA_E_ARG = 1,
  INSTA_E_CYCLE = 2,
  INSTA_E_CUDA = 3,
  INSTA_E_NOMEM = 4,
  INSTA_E_STATE = 5
} insta_status;

typedef enum { INSTA_POS = 0, INSTA_NEG = 1, INSTA_NON = 2 } insta_unate;

/* Graph description (all HOST pointers; copied by insta_graph_create).
 * Inputs are the paper's "arc attributes in consideration of rise/fall
 * conditions and unateness ... SP/EP attributes (clock arrival times, minimum
 * required times)". */
typedef struct {
  int32_t num_pins;
  int64_t num_arcs;
  const int32_t* arc_from;   /* [num_arcs] driver pin of each arc                        */
  const int32_t* arc_to;     /* [num_arcs] sink pin of each arc                          */
  const uint8_t* arc_unate;  /* [num_arcs] insta_unate                                   */
  const float* arc_mean;     /* [num_arcs][2] arc delay mean per SINK transition (Eq 1)  */
  const float* arc_sigma;    /* [num_arcs][2] arc delay std per SINK transition (Eq 2), >=0 */
  const float* src_mean;     /* [num_pins][2] or NULL(=0): arrival mean at indeg-0 pins  */
  const float* src_sigma;    /* [num_pins][2] or NULL(=0): arrival std at indeg-0 pins   */
  int32_t num_endpoints;
  const int32_t* ep_pin;     /* [num_endpoints] unique endpoint pins                     */
  const float* ep_rat;       /* [num_endpoints][2] required arrival time per rf          */
  const uint8_t* arc_class;  /* [num_arcs] 0 = net arc, 1 = cell arc, or NULL (all net);
                                used only by scenario derates (insta_forward_batch)       */
  int32_t device;            /* CUDA device ordinal                                      */
} insta_graph_desc;

/* Forward options.  n_sigma: the pessimism level of Eq 3 (3.0 in the
 * paper).  tau: 0 selects the paper's hard max (Alg 1/Alg 2 with Top-K = 1,
 * strict ">" P:L97); tau > 0 selects the LSE smooth max of Eq 4 with
 * Eq 6 gradients.  schedule (all bit-identical arrivals):
 *   0 = stage-folded persistent dataflow forward + level-synchronous sweep
 *       backward (default);
 *   1 = one launch per timing level (the paper's launch structure);
 *   2 = stage-folded persistent dataflow forward and backward (round-1 kernels);
 *   3 = level-synchronous sweep forward and backward.
 * cone_max: after insta_update_arcs(incremental = 1), the next forward takes
 * the cone pass (only heads whose inputs changed are
 * recomputed) when at most this many arcs were re-annotated, else a full pass
 * (for large batches the cone of a random update reaches every level, and the
 * dataflow full pass is faster).  0 = default limit max(64, num_arcs / 5e4) (the measured crossover);
 * < 0 = never. */
typedef struct {
  float n_sigma;
  float tau;
  int32_t want_grad_sigma; /* reserved; must be 0 in this version */
  int32_t schedule;
  int64_t cone_max;
} insta_opts;

/* Global timing metrics: WNS = min(0, min slack),
 * TNS = sum of min(0, slack) accumulated in fp64 in endpoint order. */
typedef struct {
  double wns;
  double tns;
  int32_t num_violations; /* #endpoints with slack < 0 (strict) */
  int32_t num_levels;
} insta_summary;

/* Host-only levelization (no device needed): the "topological sort" of P:L62.
 * level(p) = 0 for indeg-0 pins, else 1 + max level of its fanin sources.
 * Outputs (HOST buffers, any may be NULL): level_of_pin[num_pins];
 * order[num_pins] = caller pin at each canonical position, pins sorted by
 * (level, pin id); fanin_ptr/fanout_ptr[num_pins+1] over canonical positions;
 * fanin_arc/fanout_arc[num_arcs] caller arc ids, ascending within each row;
 * *num_levels.  INSTA_E_CYCLE on a combinational loop. */
insta_status insta_levelize(int32_t num_pins, int64_t num_arcs, const int32_t* arc_from,
                            const int32_t* arc_to, int32_t* level_of_pin, int32_t* order,
                            int32_t* fanin_ptr, int32_t* fanin_arc, int32_t* fanout_ptr,
                            int32_t* fanout_arc, int32_t* num_levels);

/* Validate, copy, levelize (host) and upload a graph; synchronous.  On success
 * *out owns every device buffer until insta_graph_destroy. */
insta_status insta_graph_create(const insta_graph_desc* desc, insta_graph** out);
void insta_graph_destroy(insta_graph* g);

/* Copy the graph's levelization to HOST buffers (same layout as
 * insta_levelize; any may be NULL); synchronous.  For bit-exact tests. */
insta_status insta_graph_export(const insta_graph* g, int32_t* level_of_pin, int32_t* order,
                                int32_t* fanin_ptr, int32_t* fanin_arc, int32_t* fanout_ptr,
                                int32_t* fanout_arc);

/* Sizes of a created graph (host). */
insta_status insta_graph_sizes(const insta_graph* g, int32_t* num_pins, int64_t* num_arcs,
                               int32_t* num_endpoints, int32_t* num_levels);

/* Schedule of the persistent passes (host; DESIGN.md §4 "stage folding"):
 * pins with one fanin and one fanout arc that are not endpoints are computed
 * inside their sink's work item, so the dependent depth is num_super_levels
 * instead of num_levels.  Reported for byte models and diagnostics. */
typedef struct {
  int32_t num_heads;          /* pins with their own work item (not folded) */
  int32_t num_super_levels;   /* dependent steps of the folded schedule */
  int64_t num_entries;        /* fanin arcs of heads (= num_arcs - num_folded) */
  int64_t num_folded;         /* folded pins */
  int64_t num_light_fanout;   /* fanout entries pulled without atomics */
  int32_t fwd_steps, bwd_steps;   /* persistent item steps per pass */
} insta_schedule;
insta_status insta_graph_schedule(const insta_graph* g, insta_schedule* out);

/* Forward: statistical arrival propagation (Eq 1-3, Alg 1 with K = 1, or
 * Eq 4) over all levels, then endpoint slack = RAT - A, min over rf (ties ->
 * R), and WNS/TNS.  o may be NULL (defaults n_sigma 3, tau 0, schedule 0).
 * out: NULL = asynchronous; non-NULL = synchronize and fill. */
insta_status insta_forward(insta_graph* g, const insta_opts* o, void* cuda_stream,
                           insta_summary* out);

/* Copy the last forward's endpoint slack (DEVICE float[num_endpoints], caller
 * endpoint order) and optionally rf_star (DEVICE uint8[num_endpoints], the rf
 * attaining the min) and the summary (forces a sync).  Any may be NULL.
 * INSTA_E_STATE if no forward since creation or since insta_update_arcs. */
insta_status insta_slack(insta_graph* g, float* slack, uint8_t* rf_star, void* cuda_stream,
                         insta_summary* out);

/* Copy the last forward's per-pin arrival state in caller pin order (DEVICE
 * buffers [num_pins][2], any may be NULL): corner arrival A = mu + n_sigma*sigma
 * (Eq 3), mean mu (Eq 1) and std sigma (Eq 2). */
insta_status insta_arrivals(insta_graph* g, float* A, float* mean, float* sigma,
                            void* cuda_stream);

/* Backward: timing gradients of L w.r.t. every arc delay mean,
 * chaining the Eq 6 softmax weights (hard mode: one-hot at the first arg-max)
 * in reverse level order.  ep_seed: DEVICE float[num_endpoints] dL/dslack, or
 * NULL for L = TNS (seed 1 where slack < 0).  d_arc_mean: DEVICE
 * float[num_arcs][2] in caller arc order, overwritten (required).
 * d_arc_sigma: DEVICE float[num_arcs][2] dL/d(arc sigma), overwritten, or NULL.
 * The sigma channel (the corner A = mu + n_sigma*sigma of
 * Eq 3 carries sigma through sqrt(sigma_j^2 + sigma_e^2) of Eq 2, and the
 * merged pin keeps the arg-max candidate's sigma, reading R1) runs
 * a separate per-level pass; d_arc_mean is bit-identical either way.
 * d_src: DEVICE float[num_pins][2] dL/d(src_mean) in caller pin order (0 at
 * non-source pins), or NULL.  Uses the tau/n_sigma of the last forward.
 * INSTA_E_STATE if the last forward is stale.  Accumulator range: every adjoint
 * is bounded by S = sum_ep |ep_seed| (TNS: S <= num_endpoints); INSTA_E_ARG
 * (nothing launched) unless S < 2^30 (schedules 0 and 3: 2^-32 fixed point in
 * int64), S < 2^18 (schedules 1 and 2: heavy-driver words fold an arrival
 * count above bit 44) or S < 2^38 (sigma channel), or if a seed is not
 * finite.  A non-NULL ep_seed costs one device reduction and a synchronization
 * for this check. */
insta_status insta_backward(insta_graph* g, const float* ep_seed, float* d_arc_mean,
                            float* d_arc_sigma, float* d_src, void* cuda_stream);

/* The TNS gradient kept current across incremental forwards (SURVEY §8(f)
 * NEXT 3: the reverse-cone backward of INSTA-Size; incremental
 * evaluation P:L229).  d_arc_mean: DEVICE float[num_arcs][2], the caller's
 * gradient buffer, owned by the caller.  The first call -- or any call after a
 * full forward, a forward with other tau / n_sigma, or with another buffer --
 * runs the full backward (default TNS seeds, as insta_backward with ep_seed =
 * NULL; also when more than max(64, num_arcs / 50000) arcs were re-annotated
 * since the snapshot: the reverse cone then spans every level and the full
 * backward is faster) and keeps a snapshot of its fixed-point adjoint sums, adjoints, seeds,
 * arg-max words and Eq 6 weights on the device (16 B + 8 B + 8 B + 4 B per work
 * head, 4 B (hard) or 32 B (LSE) per entry; allocated on first use).  A later
 * call after insta_forward cone passes only (insta_update_arcs(incremental=1)
 * below the cone threshold) re-runs the Eq 6 chain in the reverse cone of what
 * changed -- heads whose seed, arg-max or weights differ from the snapshot and,
 * level by level, every head a changed share reaches -- and updates
 * d_arc_mean in place: the buffer must still hold the previous call's result.
 * Bit-identical to insta_backward (the adjoints are integer sums of the same
 * fixed-point shares).  *incremental (HOST, may be NULL) = 1 if the update ran
 * incrementally, 0 if it ran the full backward.  Needs a schedule 0/3 forward
 * (INSTA_E_STATE otherwise); no sigma channel or source gradient. */
insta_status insta_backward_update(insta_graph* g, float* d_arc_mean, void* cuda_stream,
                                   int32_t* incremental);

/* Work heads whose Eq 6 chain the last incremental insta_backward_update re-ran
 * (HOST int64 out).  Synchronizes. */
insta_status insta_last_backward_stats(insta_graph* g, int64_t* heads_rerun);

/* Re-annotate n arcs ("re-annotate ... then re-propagate"):
 * arc_ids DEVICE int32[n] (caller ids, unique) -- or NULL with n == num_arcs
 * to re-annotate every arc in caller order -- mean/sigma DEVICE float[n][2].
 * incremental = 1: the next insta_forward recomputes only the fanout cone of
 * the changed arcs, stopping where a recomputed record does not change (a
 * dataflow pass in which pins outside the cone only republish their record;
 * same per-pin arithmetic, so results are bit-identical to a full forward);
 * 0: the next forward is a full one.  Invalid ids or
 * values are not checked on the device (caller contract). */
insta_status insta_update_arcs(insta_graph* g, int64_t n, const int32_t* arc_ids,
                               const float* mean, const float* sigma, int32_t incremental,
                               void* cuda_stream);

/* One scenario of a batched evaluation: the graph's arc
 * delays with mean and sigma of cell arcs (arc_class 1) multiplied by
 * derate_cell and of net arcs by derate_net -- materialized in fp32 as
 * fl32(x * d) -- then the listed arcs' {mean, sigma} replaced by the given
 * values (sparse overrides, e.g. a gate-sizing candidate); n_sigma is the
 * scenario's pessimism (Eq 3).  delta_* are HOST arrays, copied by the call;
 * delta arc ids must be unique within a scenario. */
typedef struct {
  float n_sigma;
  float derate_cell;
  float derate_net;
  int32_t n_delta;
  const int32_t* delta_arc;   /* HOST [n_delta] caller arc ids */
  const float* delta_mean;    /* HOST [n_delta][2] */
  const float* delta_sigma;   /* HOST [n_delta][2], >= 0 */
} insta_scenario;

/* Batched evaluation of num_scenarios independent scenarios (forward, slack,
 * WNS/TNS; optionally the TNS backward), 32 per pass with scenario-minor state.
 * Each scenario's arrivals equal insta_forward on its materialized graph bit
 * for bit.  summaries: DEVICE double[num_scenarios][3] {wns, tns,
 * num_violations}.  d_arc_mean_sum: DEVICE float[num_arcs][2], overwritten
 * with sum_s dTNS_s/d(arc mean of scenario s), or NULL for forward only.
 * tau as in insta_opts.  Does not change the graph's single-scenario state. */
insta_status insta_forward_batch(insta_graph* g, int32_t num_scenarios, const insta_scenario* sc, float tau,
                                 double* summaries, float* d_arc_mean_sum, void* cuda_stream);

/* One-cell what-if evaluation through the cone pass (SURVEY §8(f) C5 sizing
 * candidates, P:L156 INSTA-Size: "estimate the timing of each candidate"):
 * candidate i re-annotates arcs arc_ids[cand_ptr[i] .. cand_ptr[i+1]) (caller
 * ids, DEVICE int32) with mean / sigma (DEVICE float[..][2]); its summary
 * {wns, tns, num_violations} goes to summaries[i] (DEVICE double[n][3]).  Each
 * candidate is applied, evaluated with the cone pass (recomputing only what
 * its arcs reach; the endpoint slack only of the blocks it reached), and
 * reverted with a second cone pass, so the summary equals insta_forward on the
 * candidate's materialized graph bit for bit, and the graph (arrivals, slack,
 * summary) is back to its base state on return.  All candidates run inside one
 * persistent cooperative launch (grid barriers between the steps).  cand_ptr:
 * HOST int32[n + 1], ascending, cand_ptr[0] = 0.  Arc ids must lie in
 * [0, num_arcs) (device array: not checked here; the Python binding checks);
 * an arc listed twice in one candidate must carry the same record (else which
 * one applies is unspecified).  Needs a current forward of schedule 0 or 3
 * (E_STATE otherwise; uses its n_sigma / tau).  Asynchronous on cuda_stream. */
insta_status insta_eval_candidates(insta_graph* g, int32_t num_candidates, const int32_t* cand_ptr,
                                   const int32_t* arc_ids, const float* mean, const float* sigma, double* summaries,
                                   void* cuda_stream);

/* ---- Top-K unique-startpoint propagation with CPPR ----
 *
 * The paper's CPPR handling: every pin keeps, per transition rf, a
 * queue of the K largest statistical arrivals that come from DISTINCT
 * startpoints (Alg 1 l.1-18; Alg 2), and endpoint slack is
 * taken against required times "associated with respective startpoints"
 * (P:L109, L119).  Queue semantics (readings R13, R17): candidates
 * are offered in Alg 1's order (k outer, fanin arcs in caller-arc-id order,
 * s = rf before ~rf for non-unate arcs); Alg 2 replaces a queued startpoint's
 * entry only if strictly greater (then re-sorts) and inserts a new startpoint
 * only if strictly greater than the smallest entry; an empty slot has SP = -1.
 * K = 1 is the K = 1 hard merge of insta_forward (tau = 0). */

/* Per-(endpoint, startpoint) required times.  rat_ptr: HOST [num_endpoints+1]
 * row offsets (rat_ptr[0] = 0, non-decreasing); rat_sp: HOST [M] caller ids of
 * startpoint pins (indegree 0), unique within a row; rat: HOST [M][2] {R, F}
 * required times, M = rat_ptr[num_endpoints].  A startpoint missing from its
 * endpoint's row takes the endpoint's default ep_rat.  rat_ptr = NULL clears
 * the table.  Copied; synchronous.  E_ARG: malformed rows, a non-startpoint
 * pin, a duplicate, non-finite values. */
insta_status insta_set_cppr_rat(insta_graph* g, const int32_t* rat_ptr, const int32_t* rat_sp, const float* rat);

/* Top-K forward (Alg 1 + Alg 2) over all levels with the graph's current arc
 * delays; 1 <= K <= 128 (the paper's CPPR study uses K = 128), n_sigma
 * as in Eq 3.  Device state: K * 40 bytes per pin (fp64 mean and variance +
 * int32 startpoint per slot and rf; C4 at K = 128: 77 GB).  Enqueued on
 * cuda_stream.  E_ARG: K or n_sigma out of range; E_CUDA (out of memory) when
 * the queues do not fit. */
insta_status insta_topk_forward(insta_graph* g, int32_t K, float n_sigma, void* cuda_stream);

/* CPPR endpoint slack over the Top-K queues: slack(ep) = min over rf (R
 * first) and queue slots k (in order) of RAT(ep, SP_k)[rf] - A_k[rf]; the
 * first minimum wins ties.  WNS / TNS / num_violations as in insta_slack
 * (fixed-order fp64 sums).  slack: DEVICE float[num_endpoints] or NULL;
 * sp_star: DEVICE int32[num_endpoints] caller id of the critical startpoint
 * or NULL; out: summary (synchronizes) or NULL.  E_STATE without a valid
 * insta_topk_forward (insta_update_arcs invalidates it). */
insta_status insta_topk_slack(insta_graph* g, float* slack, int32_t* sp_star, void* cuda_stream, insta_summary* out);

/* The (rf, slot) of each endpoint's critical entry from the last
 * insta_topk_slack: rf_star DEVICE uint8[num_endpoints], k_star DEVICE
 * int32[num_endpoints] (either may be NULL).  E_STATE before insta_topk_slack. */
insta_status insta_topk_critical(insta_graph* g, uint8_t* rf_star, int32_t* k_star, void* cuda_stream);

/* Export of the queues in caller pin order, DEVICE arrays [num_pins][2][K]
 * (any may be NULL): A corner arrival (-inf for an empty slot), mean, sigma,
 * sp = caller id of the startpoint (-1 for an empty slot). */
insta_status insta_topk_queues(insta_graph* g, float* A, float* mean, float* sigma, int32_t* sp, void* cuda_stream);

/* ---- Clark moment-matching statistical max ----
 *
 * The north star's alternative to the paper's smooth max (Eq 4): a pin's
 * arrival per rf is the Gaussian (mu, V = sigma^2); candidates (Eq 1-2) are
 * merged by folding, in canonical candidate order (fanin arcs by caller arc
 * id, s = rf before ~rf), Clark's exact first two moments of the max of two
 * INDEPENDENT Gaussians (reading R20, correlation 0); endpoint
 * arrival A = mu + n_sigma sqrt(V) (Eq 3), slack / WNS / TNS as insta_slack.
 * fp64 state and arithmetic.  Device memory: 16 B per pin and rf + 128 B per
 * arc (fold prefixes and candidate adjoints), allocated on first use. */

/* Forward + endpoint slack; out: summary (synchronizes) or NULL. */
insta_status insta_clark_forward(insta_graph* g, float n_sigma, void* cuda_stream, insta_summary* out);

/* Results of the last insta_clark_forward, DEVICE arrays, caller order, any may
 * be NULL: A / mean / sigma float[num_pins][2]; slack float[num_endpoints];
 * rf_star uint8[num_endpoints].  E_STATE without a valid forward. */
insta_status insta_clark_results(insta_graph* g, float* A, float* mean, float* sigma, float* slack, uint8_t* rf_star,
                                 void* cuda_stream);

/* Backward of the Clark path: d_arc_mean (required) / d_arc_sigma (NULL ok)
 * DEVICE float[num_arcs][2] = dL/d(arc mean / arc sigma), d_src DEVICE
 * float[num_pins][2] = dL/d(startpoint mean) or NULL; L = TNS if ep_seed is
 * NULL, else sum_ep ep_seed[ep] * slack[ep] (ep_seed DEVICE float[num_endpoints]).
 * Reverse-level pull through Clark's Jacobian, no atomics (deterministic).
 * E_STATE without a valid insta_clark_forward (insta_update_arcs invalidates it). */
insta_status insta_clark_backward(insta_graph* g, const float* ep_seed, float* d_arc_mean, float* d_arc_sigma,
                                  float* d_src, void* cuda_stream);

/* ---- INSTA-Size device steps ----
 *
 * Stage gradient of every cell arc (arc_class 1): "the gradient sum of a cell
 * arc and its driving net arc" (R22: the driving net arc is
 * the single fanin arc of the cell arc's input pin when that pin has exactly
 * one fanin arc and it is a net arc), summed over both transitions; 0 for net
 * arcs.  d_arc_mean: DEVICE float[num_arcs][2] (e.g. insta_backward's TNS
 * gradient); stage_grad: DEVICE float[num_arcs], caller order.  E_ARG if the
 * graph was created without arc_class. */
insta_status insta_stage_gradients(insta_graph* g, const float* d_arc_mean, float* stage_grad, void* cuda_stream);

/* Threshold + rank ("Stages with gradients above a pre-defined
 * threshold are prioritized by magnitude"): the caller arc ids with
 * stage_grad < -threshold (TNS gradients are <= 0), most negative first, ties
 * in arc id order, written to out_arcs DEVICE int32[num_arcs] (entries past the
 * count are -1); out_count DEVICE int32[1].  Device-side select + stable radix
 * sort (CUB). */
insta_status insta_select_stages(insta_graph* g, const float* stage_grad, float threshold, int32_t* out_arcs,
                                 int32_t* out_count, void* cuda_stream);

/* ---- INSTA-Place timing objective (Eq 7-8) ----
 *
 * L = lambda_rc * sum over arcs k = (f -> t) of (|x_f - x_t| + |y_f - y_t|) * w_k
 * (Eq 7) with per-arc weights w_k -- the paper's "timing gradients" of the
 * critical arcs; R21: w_k = -(dTNS/dmean_R + dTNS/dmean_F) of arc k
 * (>= 0, zero for non-critical arcs), e.g. from insta_backward -- and its
 * gradient w.r.t. the pin positions (subgradient sign(0) = 0).  pin_x / pin_y:
 * DEVICE float[num_pins] caller order; arc_w: DEVICE float[num_arcs] caller
 * order; loss: DEVICE double[1] or NULL; grad_x / grad_y: DEVICE
 * float[num_pins] or both NULL.  Deterministic (fixed-order fp64 sums, pull-
 * style gradient, no atomics). */
insta_status insta_timing_loss(insta_graph* g, const float* pin_x, const float* pin_y, const float* arc_w,
                               float lambda_rc, double* loss, float* grad_x, float* grad_y, void* cuda_stream);

/* Eq 8's lambda_2 = ||a||_2 / ||b||_2 for two DEVICE float[n] gradient vectors
 * (a = the default objective's gradient, b = the timing objective's);
 * out: DEVICE double[1] (0 if ||b|| = 0).  No graph needed. */
insta_status insta_grad_norm_ratio(int64_t n, const float* a, const float* b, double* out, void* cuda_stream);

/* Statistics of the last forward: number of pins recomputed (== num_pins for a
 * full forward).  For an incremental one: the work-item heads recomputed in
 * the changed cone (insta_graph_schedule; each head's folded input pins are
 * recomputed with it).  Synchronizes. */
insta_status insta_last_forward_stats(insta_graph* g, int64_t* pins_recomputed);

/* Debug builds only (compiled with -DTK_STATS): histogram of the Top-K merge
 * batches by number of surviving candidates (33 counters, HOST output).
 * Returns 0 on success, -1 in normal builds (no counters compiled in). */
int insta_debug_topk_stats(unsigned long long* out);

/* Thread-local message for the last non-OK status ("" if none). */
const char* insta_last_error(void);

/* Library version string. */
const char* insta_version(void);

#ifdef __cplusplus
}
#endif
#endif /* INSTA_H */
