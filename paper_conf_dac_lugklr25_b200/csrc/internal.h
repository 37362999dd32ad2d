// internal.h -- device-side layout of an insta_graph (not part of the ABI).
//
// Canonical order: pins sorted by (level, caller pin id); level l occupies
// canonical positions [level_ptr[l], level_ptr[l+1]).  Level 0 holds every
// indeg-0 pin (startpoints).  Fanin arcs are stored contiguous per sink
// in canonical order ("fanin position" q), sorted by caller arc id within a
// row; this is the order the forward walks (Alg 1 l.5-7 "outPin_parent_start").
//
// Per-pin state is float4 {mu_R, mu_F, sigma_R, sigma_F} (Eq 1-2 state; the
// corner arrival A = mu + n_sigma*sigma of Eq 3 is formed on the fly), the
// same layout as an arc record {arc_mean_R, arc_mean_F, arc_std_R, arc_std_F}.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include <vector_types.h>

#include "../../include/insta.h"

namespace insta {

// fin_src word: bits 0..28 canonical source pin, bit 29 "source is a heavy
// driver" (fanout > kHeavy), bits 30..31 unateness.  Hence num_pins < 2^29.
constexpr int kUnateShift = 30;
constexpr int kHeavyFanout = 128;
constexpr int32_t kMaxPins = (1 << 29) - 1;

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

// Tiles of the persistent dataflow kernels: TILE consecutive canonical pins.
constexpr int kTile = 128;

struct DevGraph {
  int device = 0;
  int32_t n = 0, num_levels = 0, num_src = 0, num_ep = 0, num_tiles = 0;
  int64_t e = 0;
  int max_fanin = 0;
  // topology (canonical)
  int32_t* level_ptr = nullptr;    // [L+1]
  int2* tile_lv = nullptr;         // [T] {level of first pin, level of last pin}
  int32_t* level_ntiles = nullptr; // [L] tiles intersecting each level
  uint32_t* done_fwd = nullptr;    // [L] level completion counters (forward)
  uint32_t* done_bwd = nullptr;    // [L] level completion counters (backward)
  int32_t* heavy_slot = nullptr;   // [n] accumulator slot of heavy drivers, -1 otherwise
  unsigned long long* heavy_acc = nullptr;  // [num_heavy][2] fixed-point adjoints
  int32_t num_heavy = 0;
  int32_t* fanin_ptr = nullptr;    // [n+1]
  int32_t* fin_src = nullptr;      // [e] canonical source | unate << 30
  float4* fin_ms = nullptr;        // [e] {mean_R, mean_F, std_R, std_F}
  int32_t* fin_arc = nullptr;      // [e] caller arc id
  int32_t* fanout_ptr = nullptr;   // [n+1]
  int32_t* fout = nullptr;         // [e] fanin position of each fanout entry
  int32_t* arc_pos = nullptr;      // [e] caller arc id -> fanin position
  int32_t* arc_sink = nullptr;     // [e] caller arc id -> canonical sink
  int32_t* order = nullptr;        // [n] canonical -> caller pin
  float4* src_ms = nullptr;        // [num_src] source (clock) arrival distribution
  int32_t* ep_pin = nullptr;       // [P] canonical
  float2* ep_rat = nullptr;        // [P]
  uint8_t* arc_class = nullptr;    // [e] caller order (derates)
  // state
  float4* state = nullptr;         // [n]
  float2* g = nullptr;             // [e] per-fanin-arc adjoint to its source's {R, F}
  float2* seed = nullptr;          // [n] endpoint seeds (zero at non-endpoints)
  float* slack = nullptr;          // [P]
  uint8_t* rf_star = nullptr;      // [P]
  double* partials = nullptr;      // slack reduction partials
  uint32_t* ticket = nullptr;      // last-block ticket
  double* summary = nullptr;       // {wns, tns, nviol} on device
  // incremental
  uint32_t* dirty = nullptr;       // [n] stamp: pin must be recomputed in pass `inc_epoch`
  uint32_t* changed = nullptr;     // [n] stamp: pin state changed in pass `inc_epoch`
  uint32_t* tile_dirty = nullptr;  // [T] stamp: tile holds a dirty pin / produced a change
  unsigned long long* counters = nullptr;  // [4] recomputed pins etc.
  // host-side bookkeeping
  HostLevels host;
  uint32_t epoch_fwd = 0, epoch_bwd = 0, inc_epoch = 1;
  int grid_fwd = 0, grid_bwd = 0, grid_inc = 0;
  int bwd_schedule = 0;            // schedule of the last forward (backward mirrors it)
  bool fwd_valid = false;          // a forward ran since the last update
  bool pending_incremental = false;
  bool pending_full = true;
  float last_n_sigma = 3.0f, last_tau = 0.0f;
  int64_t last_recomputed = 0;
};

}  // namespace insta

struct insta_graph {
  insta::DevGraph d;
};

namespace insta {
// kernels.cu launchers; return cudaError_t as int
int launch_forward(DevGraph& g, float n_sigma, float tau, int schedule, void* stream);
int launch_forward_incremental(DevGraph& g, float n_sigma, float tau, void* stream);
int launch_slack(DevGraph& g, void* stream);
int launch_backward(DevGraph& g, const float* ep_seed, float* d_arc_mean, float* d_src,
                    void* stream);
int launch_update_arcs(DevGraph& g, int64_t n, const int32_t* ids, const float* mean,
                       const float* sigma, int incremental, void* stream);
int launch_arrivals(DevGraph& g, float* A, float* mean, float* sigma, void* stream);
int launch_copy_slack(DevGraph& g, float* slack, uint8_t* rf, void* stream);
int configure_grids(DevGraph& g);
}  // namespace insta
