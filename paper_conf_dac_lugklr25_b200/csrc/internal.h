// internal.h -- device-side layout of an insta_graph (not part of the ABI).
//
// Canonical order: pins sorted by (level, caller pin id); level l occupies
// canonical positions [level_ptr[l], level_ptr[l+1]).  Level 0 holds every
// indeg-0 pin (startpoints).  Fanin arcs are stored contiguous per sink
// in canonical order ("fanin position" q), sorted by caller arc id within a
// row; this is the order the forward walks (Alg 1 l.5-7 "outPin_parent_start").
//
// Per-pin state is 32 bytes: {double mu_R, mu_F, var_R, var_F} -- the Eq 1-2
// state (mean and variance, sigma = sqrt(var)) accumulated in fp64 (a random 32-byte gather costs
// one DRAM sector either way, and fp64 keeps 15M-pin slacks within 1e-3 ps of
// the fp64 oracle).  The least significant mantissa bit of every word carries
// the parity of the pass that wrote it (DESIGN.md §4 "dataflow"), so a reader
// knows, word by word, whether a value is from the current pass.  Arc records
// are float4 {arc_mean_R, arc_mean_F, arc_std_R, arc_std_F}.
//
// Work decomposition: every level is cut into `rounds x G`
// contiguous pin chunks of balanced work (G = resident CTAs); chunk j of level
// l is "item" (round j / G, CTA j % G).  Item descriptors are precomputed on
// the host so a CTA can prefetch the next item's topology with TMA bulk copies
// while it works on the current one.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include <vector_types.h>

#include "../../include/insta.h"

namespace insta {

// fin_src word: bits 0..28 canonical source pin, bit 29 "source is a heavy
// driver" (fanout > kHeavyFanout), bits 30..31 unateness.  num_pins < 2^29.
constexpr int kUnateShift = 30;
constexpr int kHeavyBit = 29;
constexpr int32_t kSrcMask = (1 << kHeavyBit) - 1;
constexpr int32_t kMaxPins = (1 << 29) - 1;
constexpr int kHeavyFanout = 256;
constexpr int kConeRow = 32;       // cone pass: consumer rows longer than this are not marked one by one
// ext_w word of the stage-folded schedule (fold.cpp): bit 29 "entry goes
// through a folded pin" (the heavy bit is not needed by the forward)
constexpr int kFoldBit = 29;

// CTA shape (one 1024-thread CTA per SM) and shared-memory stage capacities
// (per item; two stages are double-buffered)
constexpr int kThreads = 1024;
constexpr int kFwdPins = 1024, kFwdArcs = 1024;                     // forward item caps
constexpr int kBFwdPins = 2048, kBFwdArcs = 2048;                  // batched forward item caps
constexpr int kBwdPins = 2048, kBwdFanout = 2048, kBwdArcs = 2048;  // backward item caps
static_assert(kHeavyFanout <= kBwdFanout, "a light pin's fanout row must fit one item");

struct alignas(32) PinState {
  double mu[2];
  double var[2];
};

// item flags
constexpr int kItemDirect = 1;   // does not fit the smem stage: read topology from global
constexpr int kItemLast = 2;     // last round of its level: publish after it

// Host result of levelization (canonical layout), also what export returns.
struct HostLevels {
  int32_t n = 0;
  int64_t e = 0;
  int32_t num_levels = 0;
  std::vector<int32_t> level;       // [n] caller-indexed
  std::vector<int32_t> order;       // [n] canonical -> caller pin
  std::vector<int32_t> pos;         // [n] caller pin -> canonical
  std::vector<int32_t> level_ptr;   // [L+1]
  std::vector<int32_t> fanin_ptr;   // [n+1]
  std::vector<int32_t> fanin_arc;   // [e] caller arc id per fanin position
  std::vector<int32_t> fanout_ptr;  // [n+1]
  std::vector<int32_t> fanout_arc;  // [e] caller arc id per fanout position
};

// Returns INSTA_OK / INSTA_E_CYCLE / INSTA_E_ARG.
insta_status levelize_host(int32_t n, int64_t e, const int32_t* from, const int32_t* to,
                           HostLevels* out, std::string* err);

// Stage-folded forward schedule (fold.cpp).  "Heads" are the pins that are
// not folded, in (super-level, canonical) order; entry x of head h is the
// fanin arc e = (p -> q) of q = hd_pin[h] at row position x - hd_ptr[h]; when
// p is folded the entry also carries p's single fanin arc e' = (j -> p) and
// its source word names j.
struct FoldHost {
  std::vector<uint8_t> folded;      // [n] canonical
  std::vector<int32_t> slevel_ptr;  // [SL+1] head ranges per super-level
  std::vector<int32_t> hd_pin;      // [H] canonical pin of each head
  std::vector<int32_t> hd_ptr;      // [H+1] entry rows
  std::vector<int32_t> hd_q0;       // [H] fanin position of the head's first fanin arc
  std::vector<int32_t> hd_nfold;    // [H] folded entries (work estimate)
  std::vector<int32_t> ext_w;       // [X] source (j if folded, else p) | fold << 29 | unate(e) << 30
  std::vector<float4> ext_ms;       // [X] record of e
  std::vector<int32_t> ext_f;       // [X] folded pin p | unate(e') << 30 (folded entries)
  std::vector<float4> ext_fms;      // [X] record of e'
  std::vector<int32_t> ext_fq;      // [X] fanin position of e' (-1 if not folded)
  std::vector<int32_t> arc_xpos;    // [E] caller arc -> 2x (as e) or 2x+1 (as e')
  // backward (reverse super-level order over the same heads)
  std::vector<int32_t> hd_hslot;    // [H] heavy accumulator slot of the head (-1: light)
  std::vector<int32_t> hlfo_ptr;    // [H+1] light fanout rows of the heads
  std::vector<int32_t> hlfo;        // fanin positions (adjoint words) of those rows
  std::vector<int32_t> ext_qpos;    // [X] fanin position of e
  std::vector<int32_t> ext_bw;      // [X] fin_src word of the arc whose adjoint the entry writes (e, or e' if folded)
  std::vector<int32_t> ext_arc;     // [X] caller id of e
  std::vector<int32_t> ext_farc;    // [X] caller id of e' (-1 if not folded)
  std::vector<int32_t> ext_h;       // [X] head of each entry
  std::vector<int32_t> ep_head;     // [P] head index of each endpoint (endpoints are never folded)
  std::vector<int32_t> hd_eop;      // [H] endpoint index of each head (-1: not an endpoint)
  // incremental pass
  std::vector<int32_t> arc_head;    // [E] caller arc -> head whose item evaluates the arc
  // level-synchronous sweep (sweep.cu)
  std::vector<int32_t> ext_sh;      // [X] head index of the entry's source (j if folded, else p)
  std::vector<int32_t> hfo_ptr;     // [H+1] consumer heads of each head (deduplicated)
  std::vector<int32_t> hfo;
  std::vector<int32_t> hd_csl;      // [H] super-levels of each head's consumers: min | max << 16, -1: none
  std::vector<uint8_t> hd_hsrc;     // [H] 1: a source of the head has more than kConeRow consumers
};

// Item table: step s of CTA c is entry s * G + c.
//  forward:  a = {pin_lo, pin_hi, arc_lo, arc_hi}, b = {level, flags, 0, 0}
//  backward: a = {pin_lo, pin_hi, lfo_lo, lfo_hi}, b = {arc_lo, arc_hi, level, flags}
struct ItemTable {
  int32_t num_steps = 0;
  std::vector<int32_t> level_step0;  // [L] first step of each level (in table order)
  std::vector<int32_t> level_steps;  // [L] rounds of each level
  std::vector<int4> a, b;
};

struct DevGraph {
  int device = 0;
  int32_t n = 0, num_levels = 0, num_src = 0, num_ep = 0;
  int64_t e = 0, e_light = 0;
  int grid = 0;                    // resident CTAs (cooperative grid)
  // topology (canonical); every array is padded by >= 64 bytes for bulk copies
  int32_t* level_ptr = nullptr;    // [L+1]
  int32_t* fanin_ptr = nullptr;    // [n+1]
  int32_t* fin_src = nullptr;      // [e] canonical source | heavy << 29 | unate << 30
  float4* fin_ms = nullptr;        // [e] {mean_R, mean_F, std_R, std_F}
  int32_t* fin_arc = nullptr;      // [e] caller arc id
  int32_t* lfo_ptr = nullptr;      // [n+1] light fanout rows (heavy drivers' rows empty)
  int32_t* lfo = nullptr;          // [e_light] fanin position of each light fanout entry
  int32_t* heavy_slot = nullptr;   // [n] accumulator slot of heavy drivers, -1 otherwise
  unsigned long long* heavy_acc = nullptr;  // [num_heavy][2] fixed-point adjoints
  uint32_t* heavy_cnt = nullptr;   // [num_heavy] sink arcs that have contributed this pass
  int32_t* heavy_fo = nullptr;     // [num_heavy] fanout of each heavy driver
  int32_t num_heavy = 0;
  int32_t* arc_pos = nullptr;      // [e] caller arc id -> fanin position
  int32_t* arc_sink = nullptr;     // [e] caller arc id -> canonical sink
  int32_t* order = nullptr;        // [n] canonical -> caller pin
  float4* src_ms = nullptr;        // [num_src] source (clock) arrival distribution
  int32_t* ep_pin = nullptr;       // [P] canonical
  float2* ep_rat = nullptr;        // [P]
  uint8_t* arc_class = nullptr;    // [e] caller order (derates)
  uint8_t* fin_flags = nullptr;    // [e] fanin order: bit 0 cell arc, bit 1 overridden in the current batch
  int32_t* ep_of_pin = nullptr;    // [n] endpoint index of a canonical pin, -1 otherwise
  std::vector<int32_t> h_arc_pos;  // host copy of arc_pos (batch overrides)
  // batched scenarios (allocated on first use; scenario-minor, 32 lanes)
  PinState* b_state = nullptr;
  int32_t* b_win = nullptr;
  float4* b_wts = nullptr;
  float2* b_g = nullptr;
  unsigned long long* b_heavy = nullptr;
  // per-call scenario staging (insta_forward_batch): every micro-batch's parameters and override lists
  // packed in one pinned host buffer, moved with one H2D copy (batch_stage)
  char* b_stage = nullptr;         // device [b_stage_cap]
  void* b_stage_h = nullptr;       // pinned host [b_stage_cap]
  size_t b_stage_cap = 0;
  void* b_stage_copied = nullptr;  // cudaEvent_t: the last H2D copy out of b_stage_h finished
  void* b_stage_done = nullptr;    // cudaEvent_t: the last kernel reading b_stage finished
  float* b_slack = nullptr;
  uint8_t* b_rf = nullptr;
  double* b_partials = nullptr;
  uint32_t* b_ticket = nullptr;
  uint32_t pass_bfwd = 0, pass_bbwd = 0;
  // item tables
  int4* fwd_a = nullptr;
  int4* fwd_b = nullptr;
  int4* bfwd_a = nullptr;
  int4* bfwd_b = nullptr;
  int4* bwd_a = nullptr;
  int4* bwd_b = nullptr;
  ItemTable fwd_items, bwd_items, bfwd_items;   // bfwd: batched forward (larger caps)
  // stage-folded forward (fold.cpp)
  int32_t num_heads = 0, num_slevels = 0;
  int64_t num_ext = 0;
  int32_t* hd_pin = nullptr;
  int32_t* hd_ptr = nullptr;
  int32_t* hd_q0 = nullptr;
  int32_t* ext_w = nullptr;
  float4* ext_ms = nullptr;
  int32_t* ext_f = nullptr;
  float4* ext_fms = nullptr;
  int32_t* ext_fq = nullptr;
  int32_t* arc_xpos = nullptr;
  int4* fwdf_a = nullptr;
  int4* fwdf_b = nullptr;
  ItemTable fwdf_items;
  // stage-folded backward
  int32_t* hd_hslot = nullptr;
  int32_t* hlfo_ptr = nullptr;
  int32_t* hlfo = nullptr;
  int32_t* ext_qpos = nullptr;
  int32_t* ext_bw = nullptr;
  int32_t* ext_arc = nullptr;
  int32_t* ext_farc = nullptr;
  int32_t* ext_h = nullptr;
  int32_t* ep_head = nullptr;
  int32_t* hd_eop = nullptr;       // [H] endpoint index of each head, -1 otherwise
  uint32_t* dirty_h = nullptr;     // [H] incremental: stamp == inc epoch -> recompute
  int32_t* arc_head = nullptr;     // [E] caller arc -> head
  float2* hseed = nullptr;         // [H] endpoint seeds in head order
  // level-synchronous sweep (sweep.cu; schedule 0): one persistent launch per
  // pass, a grid barrier per super-level, one thread per head
  int sl_grid = 0, sl_grid_b = 0; // resident CTAs of the sweep forward / backward kernels
  std::vector<int32_t> h_sl_ptr;   // [SL+1] host copy of the super-level head ranges
  int32_t* sl_ptr = nullptr;       // [SL+1]
  int4* sl_slice = nullptr;        // [SL][sl_grid] per-CTA slices {a, b, xa, xb} of every super-level
  int32_t sl_max_x = 0;            // most entries in one slice (fwdx_kernel: candidate buffer size)
  // incremental backward (insta_backward_update, sweep.cu bwdi_kernel): the state of the last
  // snapshot backward -- per head its accumulated fixed-point sum and adjoint, its seed and
  // arg-max word; per entry the folded arg-max / Eq 6 weights -- and the heads touched since
  long long* acc_b = nullptr;      // [H][2]
  float2* hab_b = nullptr;         // [H]
  float2* hseed_b = nullptr;       // [H]
  int32_t* hwin_b = nullptr;       // [H]
  int32_t* fwin_b = nullptr;       // [X]
  float4* ew_b = nullptr;          // [X] (LSE)
  float4* efw_b = nullptr;         // [X] (LSE)
  uint32_t* btouch = nullptr;      // [H] == bepoch: recomputed by a cone pass since the snapshot
  uint32_t* bdirty = nullptr;      // [H] == bstamp: re-run the head's Eq 6 chain
  uint32_t* bl_cnt = nullptr;      // [SL] levels holding a dirty head
  uint32_t bepoch = 1, bstamp = 0;
  bool binc_valid = false;         // the snapshot describes the last update's gradient
  bool binc_touch_all = true;      // a full forward since the snapshot (every head may differ)
  float binc_tau = 0.f, binc_nsig = 0.f;
  float* binc_dmean = nullptr;     // the caller's gradient buffer the snapshot belongs to
  int64_t binc_heads = 0;          // heads re-run by the last update (stats)
  bool bsnap_req = false;          // the next sweep backward writes the snapshot
  int64_t binc_updates = 0;        // arcs re-annotated since the snapshot
  void* xscr = nullptr;            // fwdx_kernel: per-CTA candidate buffers for slices beyond shared memory
  int32_t* ext_sh = nullptr;       // [X] source head of each entry
  int32_t* hd_csl = nullptr;       // [H] consumer super-level range of each head
  int32_t* hfo_ptr = nullptr;      // [H+1] consumer heads of each head
  int32_t* hfo = nullptr;
  int32_t* hfo_sl = nullptr;       // super-level of each hfo entry (cone pass: the level to flag)
  uint8_t* hd_hsrc = nullptr;      // [H] a source with a long consumer row
  uint32_t* chg = nullptr;         // [n] cone pass: stamp of the pass that changed the pin's record
  long long* acc_h = nullptr;      // [H][2] fixed-point adjoint accumulators (zero between passes)
  int32_t* hwin = nullptr;         // [H] arg-max word per head (hard mode, head order)
  float4* ew = nullptr;            // [X] Eq 6 weights per entry (LSE, entry order)
  int32_t* fwin = nullptr;         // [X] arg-max word of a non-unate folded pin
  float4* efw = nullptr;           // [X] Eq 6 weights of a non-unate folded pin's arc
  uint32_t* sl_bar = nullptr;      // grid barrier counters [0..1] (reset by the last CTA of each launch)
  uint32_t* sl_cnt = nullptr;      // [SL] cone pass: dirty marks per super-level
  bool folded_valid = false;       // folded pins' records / arg-max / weights are stored (arrivals, sigma bwd)
  bool parity_mixed = false;
  bool sweep_valid = false;        // hwin / ew / fwin / efw describe every head (last full pass: schedule 0 or 3)
  bool canon_valid = false;        // win / wts (canonical) describe every pin (last full pass: schedule 1 or 2)       // a cone pass left records of different passes' parity (no dataflow pass next)
  int fwd_schedule = 0;            // schedule of the last forward
  // sigma-channel backward scratch (allocated on first use)
  void* g4 = nullptr;              // [e] float4 per fanin position
  long long* hacc4 = nullptr;      // [num_heavy][4] fixed-point adjoints
  int4* bwdf_a = nullptr;
  int4* bwdf_b = nullptr;
  ItemTable bwdf_items;
  // stage-folded batched forward
  uint8_t* ext_flags = nullptr;    // [X] bit 0 class(e) cell, bit 1 e overridden, bit 2/3 the same for e'
  std::vector<int32_t> h_arc_xpos; // host copy of arc_xpos (batch overrides)
  int4* bfwdf_a = nullptr;
  int4* bfwdf_b = nullptr;
  ItemTable bfwdf_items;
  // Top-K unique-startpoint propagation (topk.cu)
  int32_t tk_K = 0;                // queue length the buffers are sized for
  float tk_ns = 3.f;               // N_sigma of the last insta_topk_forward
  bool tk_valid = false;           // queues match the current arcs
  bool tk_slack_done = false;      // tk_slack / tk_star hold the slack of the current queues
  double2* tk_q = nullptr;         // [n][2][K] {mu, var} per queue slot (canonical pins)
  int32_t* tk_sp = nullptr;        // [n][2][K] canonical startpoint, -1 = empty slot
  int32_t* tk_list = nullptr;      // [n - num_src] per level: single-arc pins, then merging pins
  std::vector<int32_t> tk_one_ptr, tk_multi_ptr;   // [L+1] offsets of the two parts per level
  void* tk_side = nullptr;         // cudaStream_t for the single-arc part of each level
  void* tk_ev[2] = {nullptr, nullptr};   // cudaEvent_t join events
  double* tk_slack = nullptr;      // [P] CPPR slack (fp64)
  int32_t* tk_star = nullptr;      // [2][P] critical startpoint | rf << 30, slot k
  double* tk_summary = nullptr;    // {wns, tns, violations}
  // Clark moment-matching merge (clark.cu)
  void* cl_mv = nullptr;           // double2 [n][2] {mu, V}
  void* cl_pre = nullptr;          // double2 [e][2][2] fold prefix after each candidate
  void* cl_g = nullptr;            // double2 [e][2][2] candidate adjoints {mubar, Vbar}
  int32_t* cl_fo_ptr = nullptr;    // [n+1] full fanout rows
  int32_t* cl_fo_q = nullptr;      // [e] fanin position of each fanout arc
  double* cl_slack = nullptr;      // [P]
  uint8_t* cl_rf = nullptr;        // [P]
  double* cl_summary = nullptr;    // {wns, tns, violations}
  float cl_ns = 3.f;
  bool cl_valid = false;
  int32_t* cl_hv_list = nullptr;   // wide-fanout pins grouped by level
  int32_t* cl_hv_of = nullptr;     // [n] index into cl_hv_list, -1 = narrow
  void* cl_hv_sum = nullptr;       // double2 [wide][2]
  std::vector<int32_t> cl_hv_ptr;  // [L+1]
  // insta_eval_candidates: previous records of a candidate's arcs
  float* cand_old = nullptr;       // [cand_cap][4] {mean R, F, sigma R, F}
  void* elog = nullptr;            // eval_kernel undo log: changed head records / arg-max words (hard mode)
  int32_t elog_cap = 0;
  int32_t cand_cap = 0;
  // INSTA-Size selection scratch (size.cu)
  void* sz_tmp = nullptr;
  size_t sz_cap = 0;
  // Eq 7 timing objective (place.cu)
  double* tl_partials = nullptr;
  int32_t tl_cap = 0;
  int32_t* pl_ptr = nullptr;       // [n+1] incident arcs of each caller pin (fanout then fanin)
  int32_t* pl_ent = nullptr;       // [2e] other end (caller pin) | 1 << 31 if the pin is the arc's sink
  int32_t* pl_arc = nullptr;       // [2e] caller arc id
  int32_t* pl_wide = nullptr;      // caller pins with more than kPlWide incident arcs
  void* pl_xy = nullptr;           // Eq 7: positions packed per pin (scratch)
  int32_t pl_xy_cap = 0;
  int32_t num_pl_wide = -1;        // -1: not built
  // CPPR required times per (endpoint, startpoint) (insta_set_cppr_rat)
  int32_t* rat_ptr = nullptr;      // [P+1] or NULL (no table)
  int32_t* rat_sp = nullptr;       // [M] canonical startpoints, ascending within a row
  float2* rat_val = nullptr;       // [M] RAT {R, F}
  // state
  PinState* state = nullptr;       // [n]
  int32_t* win = nullptr;          // [n] hard-mode winners {R: k | s<<15, F: << 16}
  float4* wts = nullptr;           // [e] LSE weights w[rf][s] per fanin arc
  float2* g = nullptr;             // [e] per-fanin-arc adjoint to its source's {R, F} (parity LSB)
  float2* seed = nullptr;          // [n] endpoint seeds (zero at non-endpoints)
  float* slack = nullptr;          // [P]
  uint8_t* rf_star = nullptr;      // [P]
  double* partials = nullptr;      // slack reduction partials
  uint32_t* ticket = nullptr;      // last-block ticket
  double* summary = nullptr;       // {wns, tns, nviol} on device
  uint32_t* ep_blk = nullptr;      // slack blocks holding an endpoint a cone pass changed (bitmask)
  bool slack_valid = false;        // partials hold the slack blocks of the current state
  int32_t* cand_ptr_d = nullptr;   // insta_eval_candidates: device copy of cand_ptr
  int32_t cand_ptr_cap = 0;
  // incremental
  unsigned long long* counters = nullptr;  // [4] recomputed pins etc.
  // host-side bookkeeping
  HostLevels host;
  uint32_t epoch_fwd = 0, epoch_bwd = 0, inc_epoch = 0;
  uint32_t pass_fwd = 0, pass_bwd = 0;   // full passes so far; parity = pass & 1
  int bwd_schedule = 0;            // schedule of the last forward (backward mirrors it)
  bool fwd_valid = false;          // a forward ran since the last update
  bool pending_incremental = false;
  bool pending_full = true;
  int64_t pending_updates = 0;     // arcs re-annotated (incremental) since the last forward
  float last_n_sigma = 3.0f, last_tau = 0.0f;
  int64_t last_recomputed = 0;
  bool last_incremental = false;
};

// item tables (items.cpp)
void build_items(DevGraph& d, const std::vector<int32_t>& lfo_ptr);
// stage folding (fold.cpp) and its item table (items.cpp)
void build_fold(const HostLevels& h, const std::vector<int32_t>& fin_src, const std::vector<float4>& fin_ms,
                const std::vector<int32_t>& ep_of_pin, const std::vector<int32_t>& lfo_ptr,
                const std::vector<int32_t>& lfo, const std::vector<int32_t>& heavy_slot, int grid, FoldHost* out);
void build_fold_items(DevGraph& d, const FoldHost& f);

}  // namespace insta

struct insta_graph {
  insta::DevGraph d;
};

namespace insta {
// kernels.cu launchers; return cudaError_t as int
int query_grid(int device, int* grid);
int launch_forward(DevGraph& g, float n_sigma, float tau, int schedule, void* stream, int sweep_out = 0);
int launch_forward_incremental(DevGraph& g, float n_sigma, float tau, void* stream);
int launch_slack(DevGraph& g, void* stream);
int launch_backward(DevGraph& g, const float* ep_seed, float* d_arc_mean, float* d_arc_sigma, float* d_src,
                    void* stream);
int launch_gather_arcs(DevGraph& g, int n, const int32_t* ids, float* mean, float* sigma, void* stream);
// sum |ep_seed| on the device (synchronizes)
int seed_abs_sum(DevGraph& g, const float* seed, double* host_out, void* stream);
int launch_seeds(DevGraph& g, void* stream);   // TNS endpoint seeds (hseed) from the current slacks
int launch_update_arcs(DevGraph& g, int64_t n, const int32_t* ids, const float* mean,
                       const float* sigma, int incremental, void* stream);
int launch_arrivals(DevGraph& g, float* A, float* mean, float* sigma, void* stream);
// sweep.cu: level-synchronous thread-per-head passes (schedule 0)
int query_sl_grid(int device, int* grid_fwd, int* grid_bwd);
int launch_forward_sl(DevGraph& g, float n_sigma, float tau, void* stream, bool flow = false);
int launch_backward_update(DevGraph& g, float* d_arc_mean, bool snapshot_only, void* stream);
int launch_forward_cone(DevGraph& g, float n_sigma, float tau, void* stream);
int launch_eval_candidates(DevGraph& g, int num, const int32_t* cand_ptr, const int32_t* arc_ids, const float* mean,
                           const float* sigma, double* out, void* stream);
int launch_slack_delta(DevGraph& g, void* stream);
int launch_backward_sl(DevGraph& g, float* d_arc_mean, float* d_src, void* stream);
int launch_fold_fill(DevGraph& g, void* stream);   // materialize folded pins after a sweep forward
int launch_copy_slack(DevGraph& g, float* slack, uint8_t* rf, void* stream);
// batch.cu: one micro-batch of up to 32 scenarios in one pass.  All pointers are device pointers into
// the staging buffer: sc = [3][32] {n_sigma, derate_cell, derate_net}, ov_ptr = [33] per-scenario
// override ranges, ov_pos / ov_key / ov_ms = [nov] override fanin positions, entry keys, records.
struct BatchSlice {
  int nb, nov;
  const float* sc;
  const int32_t* ov_ptr;
  const int32_t* ov_pos;
  const int32_t* ov_key;
  const float4* ov_ms;
};
int launch_forward_batch(DevGraph& g, const BatchSlice& b, float tau, double* summaries, float* d_mean_sum,
                         void* stream);
int launch_topk_forward(DevGraph& g, int K, float n_sigma, void* stream);
int launch_topk_slack(DevGraph& g, float n_sigma, void* stream);
int topk_stats(unsigned long long* out);
int launch_clark_forward(DevGraph& g, float n_sigma, void* stream);
int launch_clark_backward(DevGraph& g, const float* ep_seed, float* d_mean, float* d_sigma, float* d_src,
                          void* stream);
int launch_timing_loss(DevGraph& g, const float* x, const float* y, const float* w, float lambda_rc, double* loss,
                       float* gx, float* gy, void* stream);
int launch_stage_gradients(DevGraph& g, const float* d_mean, float* out, void* stream);
int launch_select_stages(DevGraph& g, const float* grad, float threshold, int32_t* out_arcs, int32_t* out_count,
                         void* stream);
int launch_norm_ratio(int64_t n, const float* a, const float* b, double* out, void* stream);
int launch_clark_export(DevGraph& g, float* A, float* mean, float* sigma, float* slack, uint8_t* rf, void* stream);
int launch_topk_export(DevGraph& g, float* A, float* mean, float* sigma, int32_t* sp, void* stream);
int launch_topk_export_slack(DevGraph& g, float* slack, int32_t* sp_star, uint8_t* rf_star, int32_t* k_star,
                             void* stream);
// copy `bytes` of packed host data to g.b_stage (pinned bounce buffer, one async H2D copy)
int batch_stage(DevGraph& g, const void* host, size_t bytes, void* stream);
// record that every kernel reading g.b_stage has been enqueued on `stream`
int batch_stage_release(DevGraph& g, void* stream);
}  // namespace insta
