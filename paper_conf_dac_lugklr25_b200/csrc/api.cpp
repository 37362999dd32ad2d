// api.cpp -- the extern "C" boundary (include/insta.h): validation, host
// levelization, device upload, call ordering and error reporting.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "internal.h"

namespace {

thread_local std::string g_last_error;

insta_status fail(insta_status st, const std::string& msg) {
  g_last_error = msg;
  return st;
}

insta_status cuda_fail(int err, const char* where) {
  if (err == int(cudaErrorMemoryAllocation))
    return fail(INSTA_E_NOMEM, std::string(where) + ": out of device memory");
  return fail(INSTA_E_CUDA, std::string(where) + ": " +
                                cudaGetErrorString(static_cast<cudaError_t>(err)));
}

// Every device array is padded by 64 bytes: TMA bulk copies read 16-byte
// aligned windows that may extend past the last element.
template <class T>
cudaError_t upload(T** dst, const T* src, size_t count) {
  *dst = nullptr;
  size_t bytes = sizeof(T) * std::max<size_t>(count, 1) + 64;
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(dst), bytes);
  if (e != cudaSuccess) return e;
  if (count && src) return cudaMemcpy(*dst, src, sizeof(T) * count, cudaMemcpyHostToDevice);
  return cudaMemset(*dst, 0, bytes);
}

template <class T>
cudaError_t alloc_zero(T** dst, size_t count) {
  return upload<T>(dst, nullptr, count);
}

void free_graph(insta::DevGraph& d) {
  void* ptrs[] = {d.level_ptr, d.fanin_ptr, d.fin_src,   d.fin_ms,     d.fin_arc,   d.lfo_ptr,
                  d.lfo,       d.heavy_slot, d.heavy_acc, d.arc_pos,
                  d.heavy_cnt, d.heavy_fo,
                  d.arc_sink,  d.order,     d.src_ms,    d.ep_pin,     d.ep_rat,    d.arc_class,
                  d.fwd_a,     d.fwd_b,     d.bfwd_a,    d.bfwd_b,     d.bwd_a,     d.bwd_b,
                  d.state,     d.win,       d.wts,       d.g,          d.seed,      d.slack,
                  d.rf_star,   d.partials,  d.ticket,    d.summary,    d.counters,
                  d.fin_flags, d.ep_of_pin, d.b_state,   d.b_win,      d.b_wts,     d.b_g,
                  d.b_heavy,   d.b_stage,   d.b_slack,
                  d.b_rf,      d.b_partials, d.b_ticket,
                  d.hd_pin,    d.hd_ptr,    d.hd_q0,     d.ext_w,      d.ext_ms,    d.ext_f,
                  d.ext_fms,   d.ext_fq,    d.arc_xpos,  d.fwdf_a,     d.fwdf_b,    d.hd_hslot,
                  d.hlfo_ptr,  d.hlfo,      d.ext_qpos,  d.ext_bw,     d.ext_arc,   d.ext_farc,
                  d.ep_head,   d.hseed,     d.bwdf_a,    d.bwdf_b,    d.g4,        d.hacc4,
                  d.ext_flags, d.bfwdf_a,   d.bfwdf_b,   d.hd_eop,    d.dirty_h,
                  d.arc_head,  d.ext_h,     d.tk_q,      d.tk_sp,      d.tk_slack,  d.tk_star,
                  d.tk_summary, d.rat_ptr,  d.rat_sp,    d.rat_val,   d.tk_list,
                  d.cl_mv,     d.cl_pre,    d.cl_g,      d.cl_fo_ptr,  d.cl_fo_q,   d.cl_slack,
                  d.cl_rf,     d.cl_summary, d.cl_hv_list, d.cl_hv_of, d.cl_hv_sum, d.tl_partials, d.sz_tmp,
                  d.sl_ptr,    d.ext_sh,    d.hd_csl,    d.chg,       d.acc_h,     d.sl_bar,    d.sl_cnt,
                  d.hwin,      d.ew,        d.fwin,      d.efw,       d.sl_slice,  d.hfo_ptr,   d.hfo,       d.hfo_sl,    d.hd_hsrc,
                  d.cand_old,  d.elog,  d.xscr,  d.acc_b, d.hab_b, d.hseed_b, d.hwin_b, d.fwin_b, d.ew_b, d.efw_b, d.btouch, d.bdirty, d.bl_cnt, d.ep_blk,    d.cand_ptr_d, d.pl_ptr,    d.pl_ent,    d.pl_arc,    d.pl_wide,   d.pl_xy};
  for (void* p : ptrs)
    if (p) cudaFree(p);
  if (d.b_stage_h) cudaFreeHost(d.b_stage_h);
  for (void* ev : d.tk_ev)
    if (ev) cudaEventDestroy(static_cast<cudaEvent_t>(ev));
  if (d.tk_side) cudaStreamDestroy(static_cast<cudaStream_t>(d.tk_side));
  if (d.b_stage_copied) cudaEventDestroy(static_cast<cudaEvent_t>(d.b_stage_copied));
  if (d.b_stage_done) cudaEventDestroy(static_cast<cudaEvent_t>(d.b_stage_done));
}

bool finite2(const float* a, int64_t n, bool nonneg) {
  for (int64_t k = 0; k < 2 * n; ++k) {
    if (!std::isfinite(a[k])) return false;
    if (nonneg && a[k] < 0.f) return false;
  }
  return true;
}

insta_status validate_desc(const insta_graph_desc* d) {
  if (!d) return fail(INSTA_E_ARG, "graph_create: NULL descriptor");
  if (d->num_pins < 0 || d->num_arcs < 0 || d->num_endpoints < 0)
    return fail(INSTA_E_ARG, "graph_create: negative size");
  if (d->num_pins > insta::kMaxPins || d->num_arcs >= (int64_t(1) << 31))
    return fail(INSTA_E_ARG, "graph_create: size limit (num_pins < 2^29, num_arcs < 2^31)");
  if (d->num_arcs > 0 &&
      (!d->arc_from || !d->arc_to || !d->arc_unate || !d->arc_mean || !d->arc_sigma))
    return fail(INSTA_E_ARG, "graph_create: NULL arc array");
  if (d->num_endpoints > 0 && (!d->ep_pin || !d->ep_rat))
    return fail(INSTA_E_ARG, "graph_create: NULL endpoint array");
  for (int64_t a = 0; a < d->num_arcs; ++a)
    if (d->arc_unate[a] > INSTA_NON) return fail(INSTA_E_ARG, "graph_create: bad unateness");
  if (d->num_arcs > 0 && !finite2(d->arc_mean, d->num_arcs, false))
    return fail(INSTA_E_ARG, "graph_create: non-finite arc mean");
  if (d->num_arcs > 0 && !finite2(d->arc_sigma, d->num_arcs, true))
    return fail(INSTA_E_ARG, "graph_create: arc sigma must be finite and >= 0");
  if (d->src_mean && !finite2(d->src_mean, d->num_pins, false))
    return fail(INSTA_E_ARG, "graph_create: non-finite source mean");
  if (d->src_sigma && !finite2(d->src_sigma, d->num_pins, true))
    return fail(INSTA_E_ARG, "graph_create: source sigma must be finite and >= 0");
  if (d->num_endpoints > 0 && !finite2(d->ep_rat, d->num_endpoints, false))
    return fail(INSTA_E_ARG, "graph_create: non-finite required time");
  std::vector<uint8_t> seen(size_t(d->num_pins), 0);
  for (int32_t k = 0; k < d->num_endpoints; ++k) {
    int32_t p = d->ep_pin[k];
    if (p < 0 || p >= d->num_pins) return fail(INSTA_E_ARG, "graph_create: endpoint id out of range");
    if (seen[p]) return fail(INSTA_E_ARG, "graph_create: duplicate endpoint pin");
    seen[p] = 1;
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || d->device < 0 || d->device >= ndev)
    return fail(INSTA_E_ARG, "graph_create: no such CUDA device");
  return INSTA_OK;
}

}  // namespace

extern "C" {

const char* insta_last_error(void) { return g_last_error.c_str(); }

const char* insta_version(void) { return "insta-b200 0.1 (sm_100a)"; }

insta_status insta_levelize(int32_t num_pins, int64_t num_arcs, const int32_t* arc_from,
                            const int32_t* arc_to, int32_t* level_of_pin, int32_t* order,
                            int32_t* fanin_ptr, int32_t* fanin_arc, int32_t* fanout_ptr,
                            int32_t* fanout_arc, int32_t* num_levels) {
  insta::HostLevels h;
  std::string err;
  insta_status st = insta::levelize_host(num_pins, num_arcs, arc_from, arc_to, &h, &err);
  if (st != INSTA_OK) return fail(st, err);
  const size_t n = size_t(num_pins), e = size_t(num_arcs);
  if (level_of_pin) std::copy(h.level.begin(), h.level.end(), level_of_pin);
  if (order) std::copy(h.order.begin(), h.order.end(), order);
  if (fanin_ptr) std::copy(h.fanin_ptr.begin(), h.fanin_ptr.begin() + n + 1, fanin_ptr);
  if (fanout_ptr) std::copy(h.fanout_ptr.begin(), h.fanout_ptr.begin() + n + 1, fanout_ptr);
  if (fanin_arc) std::copy(h.fanin_arc.begin(), h.fanin_arc.begin() + e, fanin_arc);
  if (fanout_arc) std::copy(h.fanout_arc.begin(), h.fanout_arc.begin() + e, fanout_arc);
  if (num_levels) *num_levels = h.num_levels;
  return INSTA_OK;
}

insta_status insta_graph_create(const insta_graph_desc* desc, insta_graph** out) {
  if (!out) return fail(INSTA_E_ARG, "graph_create: NULL out");
  *out = nullptr;
  insta_status st = validate_desc(desc);
  if (st != INSTA_OK) return st;
  insta_graph* G = new (std::nothrow) insta_graph();
  if (!G) return fail(INSTA_E_NOMEM, "graph_create: host allocation");
  insta::DevGraph& d = G->d;
  d.device = desc->device;
  std::string err;
  st = insta::levelize_host(desc->num_pins, desc->num_arcs, desc->arc_from, desc->arc_to, &d.host,
                            &err);
  if (st != INSTA_OK) {
    delete G;
    return fail(st, err);
  }
  const insta::HostLevels& h = d.host;
  const int32_t n = desc->num_pins;
  const int64_t E = desc->num_arcs;
  d.n = n;
  d.e = E;
  d.num_levels = h.num_levels;
  d.num_src = n > 0 ? h.level_ptr[1] : 0;
  d.num_ep = desc->num_endpoints;

  // ---- canonical host arrays ------------------------------------------------
  const size_t nE = static_cast<size_t>(E), nN = static_cast<size_t>(n);
  std::vector<int32_t> arc_pos(nE), arc_sink(nE), fin_src(nE);
  std::vector<float4> fin_ms(nE);
  std::vector<int32_t> heavy_slot(nN, -1);
  int32_t nheavy = 0, max_fanin = 0;
  std::vector<int32_t> heavy_fo;
  for (int32_t k = 0; k < n; ++k) {
    if (h.fanout_ptr[k + 1] - h.fanout_ptr[k] > insta::kHeavyFanout) {
      heavy_slot[k] = nheavy++;
      heavy_fo.push_back(h.fanout_ptr[k + 1] - h.fanout_ptr[k]);
    }
    max_fanin = std::max(max_fanin, h.fanin_ptr[k + 1] - h.fanin_ptr[k]);
  }
  for (int32_t f : heavy_fo) {
    if (f >= (1 << 19)) {
      delete G;
      return fail(INSTA_E_ARG, "graph_create: a pin has >= 2^19 fanout arcs");
    }
  }
  if (max_fanin >= 32768) {
    delete G;
    return fail(INSTA_E_ARG, "graph_create: a pin has >= 32768 fanin arcs");
  }
  d.num_heavy = nheavy;
  for (int64_t q = 0; q < E; ++q) {
    const int32_t a = h.fanin_arc[q];
    const int32_t src = h.pos[desc->arc_from[a]];
    arc_pos[a] = int32_t(q);
    arc_sink[a] = h.pos[desc->arc_to[a]];
    fin_src[q] = src | ((heavy_slot[src] >= 0 ? 1 : 0) << insta::kHeavyBit) |
                 int32_t(uint32_t(desc->arc_unate[a]) << insta::kUnateShift);
    fin_ms[q] = make_float4(desc->arc_mean[2 * a], desc->arc_mean[2 * a + 1],
                            desc->arc_sigma[2 * a], desc->arc_sigma[2 * a + 1]);
  }
  // light fanout CSR (rows of heavy drivers left empty) and full fanout sinks
  std::vector<int32_t> lfo_ptr(nN + 1, 0), lfo;
  lfo.reserve(nE);
  for (int32_t k = 0; k < n; ++k) {
    for (int32_t r = h.fanout_ptr[k]; r < h.fanout_ptr[k + 1]; ++r) {
      const int32_t a = h.fanout_arc[r];
      if (heavy_slot[k] < 0) lfo.push_back(arc_pos[a]);
    }
    lfo_ptr[k + 1] = int32_t(lfo.size());
  }
  d.e_light = int64_t(lfo.size());
  std::vector<float4> src_ms(size_t(std::max(d.num_src, 1)));
  for (int32_t i = 0; i < d.num_src; ++i) {
    const int32_t p = h.order[i];
    src_ms[i] = make_float4(desc->src_mean ? desc->src_mean[2 * p] : 0.f,
                            desc->src_mean ? desc->src_mean[2 * p + 1] : 0.f,
                            desc->src_sigma ? desc->src_sigma[2 * p] : 0.f,
                            desc->src_sigma ? desc->src_sigma[2 * p + 1] : 0.f);
  }
  std::vector<int32_t> ep_pin(size_t(d.num_ep));
  std::vector<float2> ep_rat(size_t(d.num_ep));
  for (int32_t k = 0; k < d.num_ep; ++k) {
    ep_pin[k] = h.pos[desc->ep_pin[k]];
    ep_rat[k] = make_float2(desc->ep_rat[2 * k], desc->ep_rat[2 * k + 1]);
  }
  std::vector<uint8_t> arc_class(nE, 0);
  if (desc->arc_class) std::copy(desc->arc_class, desc->arc_class + E, arc_class.begin());
  std::vector<uint8_t> fin_flags(nE, 0);
  for (int64_t q = 0; q < E; ++q) fin_flags[q] = arc_class[h.fanin_arc[q]] ? 1 : 0;
  std::vector<int32_t> ep_of_pin(nN, -1);
  for (int32_t k = 0; k < d.num_ep; ++k) ep_of_pin[ep_pin[k]] = k;
  d.h_arc_pos = arc_pos;
  insta::FoldHost fold;
  int sms = 148;   // the sweep's grid (one CTA per SM): heads are ordered within its per-CTA slices
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, desc->device) != cudaSuccess || sms <= 0) sms = 148;
  insta::build_fold(h, fin_src, fin_ms, ep_of_pin, lfo_ptr, lfo, heavy_slot, sms, &fold);
  d.num_heads = int32_t(fold.hd_pin.size());
  d.num_slevels = int32_t(fold.slevel_ptr.size()) - 1;
  d.num_ext = int64_t(fold.ext_w.size());
  d.h_arc_xpos = fold.arc_xpos;
  std::vector<uint8_t> ext_flags(fold.ext_w.size(), 0);
  for (size_t x = 0; x < ext_flags.size(); ++x)
    ext_flags[x] = uint8_t((arc_class[fold.ext_arc[x]] ? 1 : 0) |
                           (fold.ext_farc[x] >= 0 && arc_class[fold.ext_farc[x]] ? 4 : 0));

  // ---- device: grid, items, upload ------------------------------------------------
  cudaError_t e = cudaSetDevice(d.device);
  if (e == cudaSuccess) e = static_cast<cudaError_t>(insta::query_grid(d.device, &d.grid));
  if (e == cudaSuccess) e = static_cast<cudaError_t>(insta::query_sl_grid(d.device, &d.sl_grid, &d.sl_grid_b));
  d.h_sl_ptr = fold.slevel_ptr;
  if (e == cudaSuccess) insta::build_items(d, lfo_ptr);
  if (e == cudaSuccess) insta::build_fold_items(d, fold);
  if (getenv("INSTA_DEBUG"))
    fprintf(stderr, "[insta] pins %d arcs %lld levels %d | folded %lld heads %d super-levels %d | steps: fwd %d "
            "folded fwd %d bwd %d folded bwd %d batched fwd %d\n", n, (long long)E, h.num_levels,
            (long long)(n - d.num_heads), d.num_heads, d.num_slevels, d.fwd_items.num_steps,
            d.fwdf_items.num_steps, d.bwd_items.num_steps, d.bwdf_items.num_steps, d.bfwd_items.num_steps);
#define UP(dst, src, cnt)                       \
  if (e == cudaSuccess) e = upload(&(dst), (src), size_t(cnt));
#define ZERO(dst, cnt) \
  if (e == cudaSuccess) e = alloc_zero(&(dst), size_t(cnt));
  UP(d.level_ptr, h.level_ptr.data(), h.level_ptr.size());
  UP(d.fanin_ptr, h.fanin_ptr.data(), h.fanin_ptr.size());
  UP(d.fin_src, fin_src.data(), nE);
  UP(d.fin_ms, fin_ms.data(), nE);
  UP(d.fin_arc, h.fanin_arc.data(), nE);
  UP(d.lfo_ptr, lfo_ptr.data(), lfo_ptr.size());
  UP(d.lfo, lfo.data(), lfo.size());
  UP(d.heavy_slot, heavy_slot.data(), nN);
  ZERO(d.heavy_acc, 2 * std::max(nheavy, 1));
  ZERO(d.heavy_cnt, std::max(nheavy, 1));
  UP(d.heavy_fo, heavy_fo.data(), heavy_fo.size());
  UP(d.arc_pos, arc_pos.data(), nE);
  UP(d.arc_sink, arc_sink.data(), nE);
  UP(d.order, h.order.data(), nN);
  UP(d.src_ms, src_ms.data(), src_ms.size());
  UP(d.ep_pin, ep_pin.data(), ep_pin.size());
  UP(d.ep_rat, ep_rat.data(), ep_rat.size());
  UP(d.arc_class, arc_class.data(), nE);
  UP(d.fin_flags, fin_flags.data(), nE);
  UP(d.ep_of_pin, ep_of_pin.data(), nN);
  UP(d.fwd_a, d.fwd_items.a.data(), d.fwd_items.a.size());
  UP(d.fwd_b, d.fwd_items.b.data(), d.fwd_items.b.size());
  UP(d.bfwd_a, d.bfwd_items.a.data(), d.bfwd_items.a.size());
  UP(d.bfwd_b, d.bfwd_items.b.data(), d.bfwd_items.b.size());
  UP(d.bwd_a, d.bwd_items.a.data(), d.bwd_items.a.size());
  UP(d.bwd_b, d.bwd_items.b.data(), d.bwd_items.b.size());
  UP(d.hd_pin, fold.hd_pin.data(), fold.hd_pin.size());
  UP(d.hd_ptr, fold.hd_ptr.data(), fold.hd_ptr.size());
  UP(d.hd_q0, fold.hd_q0.data(), fold.hd_q0.size());
  UP(d.ext_w, fold.ext_w.data(), fold.ext_w.size());
  UP(d.ext_ms, fold.ext_ms.data(), fold.ext_ms.size());
  UP(d.ext_f, fold.ext_f.data(), fold.ext_f.size());
  UP(d.ext_fms, fold.ext_fms.data(), fold.ext_fms.size());
  UP(d.ext_fq, fold.ext_fq.data(), fold.ext_fq.size());
  UP(d.arc_xpos, fold.arc_xpos.data(), fold.arc_xpos.size());
  UP(d.fwdf_a, d.fwdf_items.a.data(), d.fwdf_items.a.size());
  UP(d.fwdf_b, d.fwdf_items.b.data(), d.fwdf_items.b.size());
  UP(d.hd_hslot, fold.hd_hslot.data(), fold.hd_hslot.size());
  UP(d.hlfo_ptr, fold.hlfo_ptr.data(), fold.hlfo_ptr.size());
  UP(d.hlfo, fold.hlfo.data(), fold.hlfo.size());
  UP(d.ext_qpos, fold.ext_qpos.data(), fold.ext_qpos.size());
  UP(d.ext_bw, fold.ext_bw.data(), fold.ext_bw.size());
  UP(d.ext_arc, fold.ext_arc.data(), fold.ext_arc.size());
  UP(d.ext_farc, fold.ext_farc.data(), fold.ext_farc.size());
  UP(d.ext_h, fold.ext_h.data(), fold.ext_h.size());
  UP(d.ep_head, fold.ep_head.data(), fold.ep_head.size());
  UP(d.hd_eop, fold.hd_eop.data(), fold.hd_eop.size());
  ZERO(d.dirty_h, fold.hd_pin.size());
  UP(d.arc_head, fold.arc_head.data(), fold.arc_head.size());
  ZERO(d.hseed, fold.hd_pin.size());
  UP(d.bwdf_a, d.bwdf_items.a.data(), d.bwdf_items.a.size());
  UP(d.ext_flags, ext_flags.data(), ext_flags.size());
  UP(d.bfwdf_a, d.bfwdf_items.a.data(), d.bfwdf_items.a.size());
  UP(d.bfwdf_b, d.bfwdf_items.b.data(), d.bfwdf_items.b.size());
  UP(d.bwdf_b, d.bwdf_items.b.data(), d.bwdf_items.b.size());
  UP(d.sl_ptr, fold.slevel_ptr.data(), fold.slevel_ptr.size());
  {   // per-CTA slices of the sweep (sweep.cu): CTA c owns heads [lo + n c / G, lo + n (c + 1) / G)
    const int64_t G = std::max(d.sl_grid, 1);
    const int32_t SLn = d.num_slevels;
    std::vector<int4> slc(size_t(std::max<int64_t>(int64_t(SLn) * G, 1)));
    for (int32_t sv = 0; sv < SLn; ++sv) {
      const int64_t lo = fold.slevel_ptr[sv], nh = fold.slevel_ptr[sv + 1] - lo;
      for (int64_t c = 0; c < G; ++c) {
        const int32_t a = int32_t(lo + nh * c / G), b = int32_t(lo + nh * (c + 1) / G);
        slc[size_t(sv) * G + c] = make_int4(a, b, fold.hd_ptr[a], fold.hd_ptr[b]);
        if (sv > 0) d.sl_max_x = std::max(d.sl_max_x, fold.hd_ptr[b] - fold.hd_ptr[a]);
      }
    }
    UP(d.sl_slice, slc.data(), slc.size());
  }
  UP(d.ext_sh, fold.ext_sh.data(), fold.ext_sh.size());
  UP(d.hd_csl, fold.hd_csl.data(), fold.hd_csl.size());
  UP(d.hfo_ptr, fold.hfo_ptr.data(), fold.hfo_ptr.size());
  UP(d.hfo, fold.hfo.data(), fold.hfo.size());
  {   // the super-level of every consumer head in the rows (heads are in super-level order)
    std::vector<int32_t> hsl(fold.hd_pin.size(), 0), fsl(fold.hfo.size(), 0);
    for (int32_t sv = 0; sv + 1 < int32_t(fold.slevel_ptr.size()); ++sv)
      for (int32_t hh = fold.slevel_ptr[sv]; hh < fold.slevel_ptr[sv + 1]; ++hh) hsl[size_t(hh)] = sv;
    for (size_t r = 0; r < fold.hfo.size(); ++r) fsl[r] = hsl[size_t(fold.hfo[r])];
    UP(d.hfo_sl, fsl.data(), fsl.size());
  }
  UP(d.hd_hsrc, fold.hd_hsrc.data(), fold.hd_hsrc.size());
  ZERO(d.chg, nN);
  ZERO(d.acc_h, 2 * fold.hd_pin.size());
  ZERO(d.hwin, fold.hd_pin.size());
  ZERO(d.ew, fold.ext_w.size());
  ZERO(d.fwin, fold.ext_w.size());
  ZERO(d.efw, fold.ext_w.size());
  ZERO(d.sl_bar, 64);
  ZERO(d.sl_cnt, std::max<size_t>(fold.slevel_ptr.size(), 1));
  ZERO(d.state, nN);
  ZERO(d.win, nN);
  ZERO(d.wts, nE);
  ZERO(d.g, nE);
  ZERO(d.seed, nN);
  ZERO(d.slack, d.num_ep);
  ZERO(d.rf_star, d.num_ep);
  ZERO(d.partials, 3 * ((d.num_ep + 255) / 256 + 1));
  ZERO(d.ep_blk, ((d.num_ep + 255) / 256 + 1) / 32 + 1);
  ZERO(d.ticket, 1);
  ZERO(d.summary, 4);
  ZERO(d.counters, 4);
#undef UP
#undef ZERO
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    insta_status s2 = cuda_fail(int(e), "graph_create");
    free_graph(d);
    delete G;
    return s2;
  }
  *out = G;
  return INSTA_OK;
}

void insta_graph_destroy(insta_graph* g) {
  if (!g) return;
  cudaSetDevice(g->d.device);
  free_graph(g->d);
  delete g;
}

insta_status insta_graph_export(const insta_graph* g, int32_t* level_of_pin, int32_t* order,
                                int32_t* fanin_ptr, int32_t* fanin_arc, int32_t* fanout_ptr,
                                int32_t* fanout_arc) {
  if (!g) return fail(INSTA_E_ARG, "graph_export: NULL graph");
  const insta::HostLevels& h = g->d.host;
  if (level_of_pin) std::copy(h.level.begin(), h.level.end(), level_of_pin);
  if (order) std::copy(h.order.begin(), h.order.end(), order);
  if (fanin_ptr) std::copy(h.fanin_ptr.begin(), h.fanin_ptr.end(), fanin_ptr);
  if (fanout_ptr) std::copy(h.fanout_ptr.begin(), h.fanout_ptr.end(), fanout_ptr);
  if (fanin_arc) std::copy(h.fanin_arc.begin(), h.fanin_arc.end(), fanin_arc);
  if (fanout_arc) std::copy(h.fanout_arc.begin(), h.fanout_arc.end(), fanout_arc);
  return INSTA_OK;
}

insta_status insta_graph_sizes(const insta_graph* g, int32_t* num_pins, int64_t* num_arcs,
                               int32_t* num_endpoints, int32_t* num_levels) {
  if (!g) return fail(INSTA_E_ARG, "graph_sizes: NULL graph");
  if (num_pins) *num_pins = g->d.n;
  if (num_arcs) *num_arcs = g->d.e;
  if (num_endpoints) *num_endpoints = g->d.num_ep;
  if (num_levels) *num_levels = g->d.num_levels;
  return INSTA_OK;
}

insta_status insta_graph_schedule(const insta_graph* g, insta_schedule* out) {
  if (!g || !out) return fail(INSTA_E_ARG, "graph_schedule: NULL argument");
  const insta::DevGraph& d = g->d;
  out->num_heads = d.num_heads;
  out->num_super_levels = d.num_slevels;
  out->num_entries = d.num_ext;
  out->num_folded = int64_t(d.n) - d.num_heads;
  out->num_light_fanout = d.e_light;
  out->fwd_steps = d.fwdf_items.num_steps;
  out->bwd_steps = d.bwdf_items.num_steps;
  return INSTA_OK;
}

static insta_status read_summary(insta::DevGraph& d, void* stream, insta_summary* out) {
  double s[3];
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaMemcpyAsync(s, d.summary, sizeof s, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(int(e), "summary");
  out->wns = s[0];
  out->tns = s[1];
  out->num_violations = int32_t(s[2]);
  out->num_levels = d.num_levels;
  return INSTA_OK;
}

// schedule 0's full pass: 2 (default) = entry-parallel sweep without grid barriers (sweep.cu
// fwdx_kernel, parity dataflow), 1 = the same with level barriers, 0 = the warp-round dataflow
// kernel of schedule 2 (kernels.cu); INSTA_FWDX overrides (measurements only)
static int fwdx_mode() {
  static int m = -1;
  if (m < 0) {
    const char* v = getenv("INSTA_FWDX");
    m = v ? atoi(v) : 2;
  }
  return m;
}

insta_status insta_forward(insta_graph* g, const insta_opts* o, void* cuda_stream,
                           insta_summary* out) {
  if (!g) return fail(INSTA_E_ARG, "forward: NULL graph");
  insta_opts opt{3.0f, 0.0f, 0, 0, 0};
  if (o) opt = *o;
  if (!std::isfinite(opt.n_sigma) || opt.n_sigma < 0.f || !std::isfinite(opt.tau) ||
      opt.tau < 0.f)
    return fail(INSTA_E_ARG, "forward: n_sigma and tau must be finite and >= 0");
  if (opt.want_grad_sigma != 0) return fail(INSTA_E_ARG, "forward: want_grad_sigma unsupported");
  if (opt.schedule < 0 || opt.schedule > 3) return fail(INSTA_E_ARG, "forward: bad schedule");
  insta::DevGraph& d = g->d;
  cudaSetDevice(d.device);
  // incremental cone pass when only incremental updates happened since a
  // forward with the same options (schedules 0, 2 and 3)
  // (the cone pass keeps the previous pass's records, arg-max and weights of clean heads: they
  // must be in the layout this schedule's backward reads -- head/entry order for 0 and 3,
  // canonical for 2)
  const bool sweep_sched = opt.schedule == 0 || opt.schedule == 3;
  const int64_t cone_max = opt.cone_max != 0 ? opt.cone_max : std::max<int64_t>(64, d.e / 50000);   // crossover measured: tools/cone_cross.py
  const bool inc = d.pending_incremental && !d.pending_full && opt.schedule != 1 &&
                   opt.n_sigma == d.last_n_sigma && opt.tau == d.last_tau &&
                   (sweep_sched ? d.sweep_valid && d.pending_updates <= cone_max : d.canon_valid);
  int err = 0;
  if ((opt.schedule == 0 || opt.schedule == 3) && inc) {   // cone pass (sweep.cu)
    err = insta::launch_forward_cone(d, opt.n_sigma, opt.tau, cuda_stream);
    if (!err) {
      d.last_n_sigma = opt.n_sigma;
      d.last_tau = opt.tau;
      err = insta::launch_slack_delta(d, cuda_stream);   // only the slack blocks the cone reached
    }
  } else if (opt.schedule == 3 || (opt.schedule == 0 && (d.parity_mixed || fwdx_mode() != 0))) {
    // entry-parallel sweep forward (sweep.cu fwdx_kernel): level barriers for schedule 3 and
    // right after a cone pass (mixed record parity cannot order a dataflow pass)
    const bool flow = opt.schedule == 0 && !d.parity_mixed && fwdx_mode() == 2;
    err = insta::launch_forward_sl(d, opt.n_sigma, opt.tau, cuda_stream, flow);
    if (!err) {
      d.last_n_sigma = opt.n_sigma;
      d.last_tau = opt.tau;
      err = insta::launch_slack(d, cuda_stream);
    }
  } else if (opt.schedule == 0) {   // stage-folded dataflow forward writing the sweep backward's inputs
    err = insta::launch_forward(d, opt.n_sigma, opt.tau, 0, cuda_stream, 1);
  } else if (inc && !d.parity_mixed) {   // schedule 2: dataflow incremental pass over every head
    err = insta::launch_forward_incremental(d, opt.n_sigma, opt.tau, cuda_stream);
  } else {   // 1: one launch per level; 2: persistent dataflow (kernels.cu); both store every record
    // (schedule 2 orders by parity: after a sweep cone pass the parity is mixed -> per-level launches once)
    const int ks = (opt.schedule == 2 && !d.parity_mixed) ? 0 : 1;
    err = insta::launch_forward(d, opt.n_sigma, opt.tau, ks, cuda_stream);
    if (!err) d.parity_mixed = false;
  }
  if (err) return cuda_fail(err, "forward");
  if (!inc) {
    d.binc_touch_all = true;   // every head's arg-max / weights may differ from the backward snapshot
    d.sweep_valid = sweep_sched;
    d.canon_valid = !sweep_sched;
  } else if (sweep_sched) {
    d.canon_valid = false;
  } else {
    d.sweep_valid = false;
  }
  d.bwd_schedule = opt.schedule;
  d.fwd_schedule = opt.schedule;
  d.fwd_valid = true;
  d.pending_full = false;
  d.pending_incremental = false;
  d.pending_updates = 0;
  d.last_incremental = inc;
  d.last_recomputed = d.n;
  if (out) return read_summary(d, cuda_stream, out);
  return INSTA_OK;
}

insta_status insta_slack(insta_graph* g, float* slack, uint8_t* rf_star, void* cuda_stream,
                         insta_summary* out) {
  if (!g) return fail(INSTA_E_ARG, "slack: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d.fwd_valid) return fail(INSTA_E_STATE, "slack: no valid forward (call insta_forward)");
  cudaSetDevice(d.device);
  int err = insta::launch_copy_slack(d, slack, rf_star, cuda_stream);
  if (err) return cuda_fail(err, "slack");
  if (out) return read_summary(d, cuda_stream, out);
  return INSTA_OK;
}

insta_status insta_arrivals(insta_graph* g, float* A, float* mean, float* sigma,
                            void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "arrivals: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d.fwd_valid) return fail(INSTA_E_STATE, "arrivals: no valid forward");
  cudaSetDevice(d.device);
  int err = insta::launch_arrivals(d, A, mean, sigma, cuda_stream);
  if (err) return cuda_fail(err, "arrivals");
  return INSTA_OK;
}

insta_status insta_backward(insta_graph* g, const float* ep_seed, float* d_arc_mean,
                            float* d_arc_sigma, float* d_src, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "backward: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d_arc_mean && d.e > 0) return fail(INSTA_E_ARG, "backward: d_arc_mean is required");
  if (!d.fwd_valid) return fail(INSTA_E_STATE, "backward: no valid forward (call insta_forward)");
  cudaSetDevice(d.device);
  // accumulator range (include/insta.h): every adjoint is bounded by sum |ep_seed|
  // (TNS: the number of violating endpoints <= num_endpoints).  The sweep backward
  // accumulates 2^-32 fixed point in int64; schedules 1 and 2 fold an arrival count
  // into the words of heavy drivers (2^-24 units below bit 44); the sigma channel
  // accumulates 2^-24 fixed point in int64.
  const double limit = d_arc_sigma ? 0x1p38 : (d.bwd_schedule == 0 || d.bwd_schedule == 3) ? 0x1p30 : 0x1p18;
  if (ep_seed) {
    double sum = 0.0;
    const int e2 = insta::seed_abs_sum(d, ep_seed, &sum, cuda_stream);
    if (e2) return cuda_fail(e2, "backward");
    if (!(sum < limit)) {
      char msg[160];
      snprintf(msg, sizeof msg, "backward: sum |ep_seed| = %g is not finite or exceeds the adjoint bound %g", sum,
               limit);
      return fail(INSTA_E_ARG, msg);
    }
  } else if (double(d.num_ep) >= limit) {
    return fail(INSTA_E_ARG, "backward: too many endpoints for this schedule's accumulators (use schedule 0)");
  }
  int err = insta::launch_backward(d, ep_seed, d_arc_mean, d_arc_sigma, d_src, cuda_stream);
  if (err) return cuda_fail(err, "backward");
  return INSTA_OK;
}

insta_status insta_backward_update(insta_graph* g, float* d_arc_mean, void* cuda_stream, int32_t* incremental) {
  if (!g) return fail(INSTA_E_ARG, "backward_update: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d_arc_mean && d.e > 0) return fail(INSTA_E_ARG, "backward_update: d_arc_mean is required");
  if (!d.fwd_valid) return fail(INSTA_E_STATE, "backward_update: no valid forward (call insta_forward)");
  if (d.bwd_schedule != 0 && d.bwd_schedule != 3)
    return fail(INSTA_E_STATE, "backward_update: needs a schedule-0/3 forward (the sweep backward's accumulators)");
  if (double(d.num_ep) >= 0x1p30)
    return fail(INSTA_E_ARG, "backward_update: too many endpoints for the sweep accumulators");
  cudaSetDevice(d.device);
  // incremental only from a snapshot of the same buffer and options, with cone passes only since
  // and few re-annotated arcs: the reverse cone costs a grid barrier per super-level it spans,
  // so past ~E/5e4 updated arcs (C4: 426) the full backward is the faster one (bench
  // incremental.C4_backward_update: 1e-5 of the arcs 0.10 vs 0.37 ms, 1e-4 0.49 vs 0.37 ms)
  const int64_t upd_max = std::max<int64_t>(64, d.e / 50000);
  const bool full = !d.binc_valid || d.binc_touch_all || d.binc_dmean != d_arc_mean ||
                    d.binc_tau != d.last_tau || d.binc_nsig != d.last_n_sigma || d.binc_updates > upd_max;
  int err = insta::launch_backward_update(d, d_arc_mean, full, cuda_stream);
  if (err) {
    d.binc_valid = false;
    return cuda_fail(err, "backward_update");
  }
  d.binc_valid = true;
  d.binc_touch_all = false;
  d.binc_updates = 0;
  d.binc_dmean = d_arc_mean;
  d.binc_tau = d.last_tau;
  d.binc_nsig = d.last_n_sigma;
  if (incremental) *incremental = full ? 0 : 1;
  return INSTA_OK;
}

insta_status insta_last_backward_stats(insta_graph* g, int64_t* heads_rerun) {
  if (!g || !heads_rerun) return fail(INSTA_E_ARG, "last_backward_stats: NULL argument");
  insta::DevGraph& d = g->d;
  unsigned long long v = 0;
  const cudaError_t e = cudaMemcpy(&v, d.counters + 2, sizeof v, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return cuda_fail(int(e), "last_backward_stats");
  *heads_rerun = int64_t(v);
  return INSTA_OK;
}

insta_status insta_update_arcs(insta_graph* g, int64_t n, const int32_t* arc_ids,
                               const float* mean, const float* sigma, int32_t incremental,
                               void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "update_arcs: NULL graph");
  insta::DevGraph& d = g->d;
  if (n < 0 || (n > 0 && (!mean || !sigma)) || (n > 0 && !arc_ids && n != d.e))
    return fail(INSTA_E_ARG, "update_arcs: bad arguments (arc_ids may be NULL only with n == num_arcs)");
  if (n > d.e) return fail(INSTA_E_ARG, "update_arcs: more updates than arcs");
  cudaSetDevice(d.device);
  int err = insta::launch_update_arcs(d, n, arc_ids, mean, sigma, incremental, cuda_stream);
  if (err) return cuda_fail(err, "update_arcs");
  d.fwd_valid = false;
  d.tk_valid = false;
  d.cl_valid = false;
  if (incremental && !d.pending_full) d.pending_incremental = true;
  else d.pending_full = true;
  d.pending_updates += n;
  d.binc_updates += n;
  return INSTA_OK;
}

insta_status insta_eval_candidates(insta_graph* g, int32_t num_candidates, const int32_t* cand_ptr,
                                   const int32_t* arc_ids, const float* mean, const float* sigma, double* summaries,
                                   void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "eval_candidates: NULL graph");
  insta::DevGraph& d = g->d;
  if (num_candidates < 0 || (num_candidates > 0 && (!cand_ptr || !summaries)))
    return fail(INSTA_E_ARG, "eval_candidates: bad arguments");
  if (!d.fwd_valid || d.pending_full || d.pending_incremental || !d.sweep_valid)
    return fail(INSTA_E_STATE, "eval_candidates: needs a current schedule-0/3 forward (call insta_forward)");
  int32_t maxn = 0;
  for (int32_t i = 0; i < num_candidates; ++i) {
    const int32_t n = cand_ptr[i + 1] - cand_ptr[i];
    if (n < 0 || cand_ptr[i] < 0) return fail(INSTA_E_ARG, "eval_candidates: cand_ptr not ascending");
    maxn = std::max(maxn, n);
  }
  if (maxn > 0 && (!arc_ids || !mean || !sigma)) return fail(INSTA_E_ARG, "eval_candidates: NULL arc arrays");
  cudaSetDevice(d.device);
  if (num_candidates == 0) return INSTA_OK;
  if (cand_ptr[0] != 0) return fail(INSTA_E_ARG, "eval_candidates: cand_ptr[0] must be 0");
  if (!d.slack_valid) {   // the base slack blocks the kernel updates in place
    const int err = insta::launch_slack(d, cuda_stream);
    if (err) return cuda_fail(err, "eval_candidates");
  }
  // every candidate applied, evaluated and reverted inside one persistent launch (sweep.cu
  // eval_kernel); on return the graph, its slack and summary are the base state bit for bit
  const int err = insta::launch_eval_candidates(d, num_candidates, cand_ptr, arc_ids, mean, sigma, summaries,
                                                cuda_stream);
  if (err) {
    d.fwd_valid = false;
    d.pending_full = true;
    return cuda_fail(err, "eval_candidates");
  }
  d.pending_updates = 0;
  return INSTA_OK;
}

insta_status insta_forward_batch(insta_graph* g, int32_t num_scenarios, const insta_scenario* sc, float tau,
                                 double* summaries, float* d_arc_mean_sum, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "forward_batch: NULL graph");
  if (num_scenarios < 0 || (num_scenarios > 0 && (!sc || !summaries)))
    return fail(INSTA_E_ARG, "forward_batch: bad arguments");
  if (!std::isfinite(tau) || tau < 0.f) return fail(INSTA_E_ARG, "forward_batch: tau must be >= 0");
  insta::DevGraph& d = g->d;
  for (int32_t s = 0; s < num_scenarios; ++s) {
    const insta_scenario& x = sc[s];
    if (!std::isfinite(x.n_sigma) || x.n_sigma < 0.f || !std::isfinite(x.derate_cell) || x.derate_cell < 0.f ||
        !std::isfinite(x.derate_net) || x.derate_net < 0.f)
      return fail(INSTA_E_ARG, "forward_batch: scenario n_sigma and derates must be finite and >= 0");
    if (x.n_delta < 0 || (x.n_delta > 0 && (!x.delta_arc || !x.delta_mean || !x.delta_sigma)))
      return fail(INSTA_E_ARG, "forward_batch: bad scenario delta list");
    for (int32_t k = 0; k < x.n_delta; ++k) {
      if (x.delta_arc[k] < 0 || x.delta_arc[k] >= d.e) return fail(INSTA_E_ARG, "forward_batch: delta arc out of range");
      for (int r = 0; r < 2; ++r)
        if (!std::isfinite(x.delta_mean[2 * k + r]) || !std::isfinite(x.delta_sigma[2 * k + r]) ||
            x.delta_sigma[2 * k + r] < 0.f)
          return fail(INSTA_E_ARG, "forward_batch: bad delta value");
    }
  }
  cudaSetDevice(d.device);
  cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
  if (d_arc_mean_sum && d.num_ep >= (1 << 19))   // batched backward: count-folded heavy accumulators (TNS seeds)
    return fail(INSTA_E_ARG, "forward_batch: gradients need num_endpoints < 2^19 (heavy accumulator range)");
  if (d_arc_mean_sum && d.e > 0) {
    cudaError_t e = cudaMemsetAsync(d_arc_mean_sum, 0, sizeof(float) * 2 * size_t(d.e), st);
    if (e != cudaSuccess) return cuda_fail(int(e), "forward_batch");
  }
  // Pack every micro-batch of 32 scenarios: [3][32] parameters, [33] override ranges, then the
  // override fanin positions, entry keys and records of all micro-batches (one H2D copy).
  constexpr int kL = 32;
  const int nm = (num_scenarios + kL - 1) / kL;
  int64_t nov_all = 0;
  for (int32_t s = 0; s < num_scenarios; ++s) nov_all += sc[s].n_delta;
  const size_t head = size_t(nm) * (3 * kL + kL + 1) * 4;
  const size_t o_pos = (head + 15) & ~size_t(15);
  const size_t o_key = o_pos + ((size_t(nov_all) * 4 + 15) & ~size_t(15));
  const size_t o_ms = o_key + ((size_t(nov_all) * 4 + 15) & ~size_t(15));
  const size_t bytes = o_ms + size_t(nov_all) * 16;
  std::vector<char> buf(bytes);
  int64_t nov = 0;
  std::vector<int> nov_of(nm), first_of(nm);
  for (int m = 0; m < nm; ++m) {
    float* par = reinterpret_cast<float*>(buf.data() + size_t(m) * (4 * kL + 1) * 4);
    int32_t* ovp = reinterpret_cast<int32_t*>(par + 3 * kL);
    first_of[m] = int(nov);
    ovp[0] = 0;
    for (int s = 0; s < kL; ++s) {
      const int b = m * kL + s;
      const insta_scenario* x = b < num_scenarios ? &sc[b] : nullptr;
      par[s] = x ? x->n_sigma : 0.f;
      par[kL + s] = x ? x->derate_cell : 1.f;
      par[2 * kL + s] = x ? x->derate_net : 1.f;
      for (int32_t k = 0; x && k < x->n_delta; ++k, ++nov) {
        reinterpret_cast<int32_t*>(buf.data() + o_pos)[nov] = d.h_arc_pos[x->delta_arc[k]];
        reinterpret_cast<int32_t*>(buf.data() + o_key)[nov] = d.h_arc_xpos[x->delta_arc[k]];
        reinterpret_cast<float4*>(buf.data() + o_ms)[nov] =
            make_float4(x->delta_mean[2 * k], x->delta_mean[2 * k + 1], x->delta_sigma[2 * k], x->delta_sigma[2 * k + 1]);
      }
      ovp[s + 1] = int32_t(nov - first_of[m]);
    }
    nov_of[m] = int(nov - first_of[m]);
  }
  int err = insta::batch_stage(d, buf.data(), bytes, cuda_stream);
  if (err) return cuda_fail(err, "forward_batch");
  for (int m = 0; m < nm; ++m) {
    const char* dev = d.b_stage;
    insta::BatchSlice b;
    b.nb = std::min(kL, num_scenarios - m * kL);
    b.nov = nov_of[m];
    b.sc = reinterpret_cast<const float*>(dev + size_t(m) * (4 * kL + 1) * 4);
    b.ov_ptr = reinterpret_cast<const int32_t*>(b.sc + 3 * kL);
    b.ov_pos = reinterpret_cast<const int32_t*>(dev + o_pos) + first_of[m];
    b.ov_key = reinterpret_cast<const int32_t*>(dev + o_key) + first_of[m];
    b.ov_ms = reinterpret_cast<const float4*>(dev + o_ms) + first_of[m];
    err = insta::launch_forward_batch(d, b, tau, summaries + 3 * size_t(m) * kL, d_arc_mean_sum, cuda_stream);
    if (err) return cuda_fail(err, "forward_batch");
  }
  err = insta::batch_stage_release(d, cuda_stream);
  if (err) return cuda_fail(err, "forward_batch");
  return INSTA_OK;
}

// ---------------------------------------------------------------------------
// Top-K unique-startpoint propagation and CPPR slack
// ---------------------------------------------------------------------------
insta_status insta_set_cppr_rat(insta_graph* g, const int32_t* rat_ptr, const int32_t* rat_sp, const float* rat) {
  if (!g) return fail(INSTA_E_ARG, "set_cppr_rat: NULL graph");
  insta::DevGraph& d = g->d;
  cudaSetDevice(d.device);
  if (d.rat_ptr) cudaFree(d.rat_ptr);
  if (d.rat_sp) cudaFree(d.rat_sp);
  if (d.rat_val) cudaFree(d.rat_val);
  d.rat_ptr = nullptr;
  d.rat_sp = nullptr;
  d.rat_val = nullptr;
  d.tk_slack_done = false;
  if (!rat_ptr) return INSTA_OK;   // table cleared: every startpoint takes the default RAT
  const int32_t P = d.num_ep;
  if (rat_ptr[0] != 0) return fail(INSTA_E_ARG, "set_cppr_rat: rat_ptr[0] must be 0");
  for (int32_t e = 0; e < P; ++e)
    if (rat_ptr[e + 1] < rat_ptr[e]) return fail(INSTA_E_ARG, "set_cppr_rat: rat_ptr must be non-decreasing");
  const int32_t M = rat_ptr[P];
  if (M > 0 && (!rat_sp || !rat)) return fail(INSTA_E_ARG, "set_cppr_rat: NULL table");
  std::vector<std::pair<int32_t, int32_t>> row;
  std::vector<int32_t> sp(size_t(std::max(M, 1)));
  std::vector<float2> val(size_t(std::max(M, 1)));
  for (int32_t e = 0; e < P; ++e) {
    row.clear();
    for (int32_t m = rat_ptr[e]; m < rat_ptr[e + 1]; ++m) {
      const int32_t p = rat_sp[m];
      if (p < 0 || p >= d.n) return fail(INSTA_E_ARG, "set_cppr_rat: startpoint id out of range");
      const int32_t c = d.host.pos[p];
      if (c >= d.num_src) return fail(INSTA_E_ARG, "set_cppr_rat: pin is not a startpoint (has fanin)");
      if (!std::isfinite(rat[2 * size_t(m)]) || !std::isfinite(rat[2 * size_t(m) + 1]))
        return fail(INSTA_E_ARG, "set_cppr_rat: non-finite required time");
      row.emplace_back(c, m);
    }
    std::sort(row.begin(), row.end());
    for (size_t k = 0; k < row.size(); ++k) {
      if (k && row[k].first == row[k - 1].first) return fail(INSTA_E_ARG, "set_cppr_rat: duplicate startpoint in a row");
      sp[rat_ptr[e] + k] = row[k].first;
      val[rat_ptr[e] + k] = make_float2(rat[2 * size_t(row[k].second)], rat[2 * size_t(row[k].second) + 1]);
    }
  }
  cudaError_t e = cudaMalloc(&d.rat_ptr, sizeof(int32_t) * (size_t(P) + 1));
  if (e == cudaSuccess) e = cudaMalloc(&d.rat_sp, sizeof(int32_t) * sp.size());
  if (e == cudaSuccess) e = cudaMalloc(&d.rat_val, sizeof(float2) * val.size());
  if (e == cudaSuccess) e = cudaMemcpy(d.rat_ptr, rat_ptr, sizeof(int32_t) * (size_t(P) + 1), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(d.rat_sp, sp.data(), sizeof(int32_t) * sp.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(d.rat_val, val.data(), sizeof(float2) * val.size(), cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return cuda_fail(int(e), "set_cppr_rat");
  return INSTA_OK;
}

insta_status insta_topk_forward(insta_graph* g, int32_t K, float n_sigma, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "topk_forward: NULL graph");
  if (K < 1 || K > 128) return fail(INSTA_E_ARG, "topk_forward: K must be in [1, 128]");
  if (!std::isfinite(n_sigma) || n_sigma < 0.f) return fail(INSTA_E_ARG, "topk_forward: n_sigma must be >= 0");
  insta::DevGraph& d = g->d;
  cudaSetDevice(d.device);
  int err = insta::launch_topk_forward(d, K, n_sigma, cuda_stream);
  if (err) return cuda_fail(err, "topk_forward");
  d.tk_ns = n_sigma;
  d.tk_valid = true;
  d.tk_slack_done = false;
  return INSTA_OK;
}

insta_status insta_topk_slack(insta_graph* g, float* slack, int32_t* sp_star, void* cuda_stream, insta_summary* out) {
  if (!g) return fail(INSTA_E_ARG, "topk_slack: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d.tk_valid) return fail(INSTA_E_STATE, "topk_slack: no valid Top-K forward (call insta_topk_forward)");
  cudaSetDevice(d.device);
  int err = insta::launch_topk_slack(d, d.tk_ns, cuda_stream);
  if (!err && (slack || sp_star)) err = insta::launch_topk_export_slack(d, slack, sp_star, nullptr, nullptr, cuda_stream);
  if (err) return cuda_fail(err, "topk_slack");
  d.tk_slack_done = true;
  if (out) {
    double s[3];
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    cudaError_t e = cudaMemcpyAsync(s, d.tk_summary, sizeof s, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(int(e), "topk_slack");
    out->wns = s[0];
    out->tns = s[1];
    out->num_violations = int32_t(s[2]);
    out->num_levels = d.num_levels;
  }
  return INSTA_OK;
}

insta_status insta_topk_critical(insta_graph* g, uint8_t* rf_star, int32_t* k_star, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "topk_critical: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d.tk_valid || !d.tk_slack_done) return fail(INSTA_E_STATE, "topk_critical: call insta_topk_slack first");
  cudaSetDevice(d.device);
  int err = insta::launch_topk_export_slack(d, nullptr, nullptr, rf_star, k_star, cuda_stream);
  if (err) return cuda_fail(err, "topk_critical");
  return INSTA_OK;
}

insta_status insta_topk_queues(insta_graph* g, float* A, float* mean, float* sigma, int32_t* sp, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "topk_queues: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d.tk_valid) return fail(INSTA_E_STATE, "topk_queues: no valid Top-K forward (call insta_topk_forward)");
  cudaSetDevice(d.device);
  int err = insta::launch_topk_export(d, A, mean, sigma, sp, cuda_stream);
  if (err) return cuda_fail(err, "topk_queues");
  return INSTA_OK;
}

// ---------------------------------------------------------------------------
// Clark moment-matching merge
// ---------------------------------------------------------------------------
insta_status insta_clark_forward(insta_graph* g, float n_sigma, void* cuda_stream, insta_summary* out) {
  if (!g) return fail(INSTA_E_ARG, "clark_forward: NULL graph");
  if (!std::isfinite(n_sigma) || n_sigma < 0.f) return fail(INSTA_E_ARG, "clark_forward: n_sigma must be >= 0");
  insta::DevGraph& d = g->d;
  cudaSetDevice(d.device);
  int err = insta::launch_clark_forward(d, n_sigma, cuda_stream);
  if (err) return cuda_fail(err, "clark_forward");
  d.cl_ns = n_sigma;
  d.cl_valid = true;
  if (out) {
    double s[3];
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    cudaError_t e = cudaMemcpyAsync(s, d.cl_summary, sizeof s, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(int(e), "clark_forward");
    out->wns = s[0];
    out->tns = s[1];
    out->num_violations = int32_t(s[2]);
    out->num_levels = d.num_levels;
  }
  return INSTA_OK;
}

insta_status insta_clark_results(insta_graph* g, float* A, float* mean, float* sigma, float* slack, uint8_t* rf_star,
                                 void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "clark_results: NULL graph");
  insta::DevGraph& d = g->d;
  if (!d.cl_valid) return fail(INSTA_E_STATE, "clark_results: no valid insta_clark_forward");
  cudaSetDevice(d.device);
  int err = insta::launch_clark_export(d, A, mean, sigma, slack, rf_star, cuda_stream);
  if (err) return cuda_fail(err, "clark_results");
  return INSTA_OK;
}

insta_status insta_clark_backward(insta_graph* g, const float* ep_seed, float* d_arc_mean, float* d_arc_sigma,
                                  float* d_src, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "clark_backward: NULL graph");
  if (!d_arc_mean && g->d.e > 0) return fail(INSTA_E_ARG, "clark_backward: NULL d_arc_mean");
  insta::DevGraph& d = g->d;
  if (!d.cl_valid) return fail(INSTA_E_STATE, "clark_backward: no valid insta_clark_forward");
  cudaSetDevice(d.device);
  int err = insta::launch_clark_backward(d, ep_seed, d_arc_mean, d_arc_sigma, d_src, cuda_stream);
  if (err) return cuda_fail(err, "clark_backward");
  return INSTA_OK;
}

// ---------------------------------------------------------------------------
// INSTA-Place timing objective, Eq 7 / Eq 8
// ---------------------------------------------------------------------------
insta_status insta_timing_loss(insta_graph* g, const float* pin_x, const float* pin_y, const float* arc_w,
                               float lambda_rc, double* loss, float* grad_x, float* grad_y, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "timing_loss: NULL graph");
  insta::DevGraph& d = g->d;
  if (d.n > 0 && (!pin_x || !pin_y)) return fail(INSTA_E_ARG, "timing_loss: NULL pin positions");
  if (d.e > 0 && !arc_w) return fail(INSTA_E_ARG, "timing_loss: NULL arc weights");
  if ((grad_x == nullptr) != (grad_y == nullptr)) return fail(INSTA_E_ARG, "timing_loss: grad_x and grad_y go together");
  if (!std::isfinite(lambda_rc)) return fail(INSTA_E_ARG, "timing_loss: lambda_rc must be finite");
  cudaSetDevice(d.device);
  int err = insta::launch_timing_loss(d, pin_x, pin_y, arc_w, lambda_rc, loss, grad_x, grad_y, cuda_stream);
  if (err) return cuda_fail(err, "timing_loss");
  return INSTA_OK;
}

insta_status insta_grad_norm_ratio(int64_t n, const float* a, const float* b, double* out, void* cuda_stream) {
  if (n < 0 || !out || (n > 0 && (!a || !b))) return fail(INSTA_E_ARG, "grad_norm_ratio: bad arguments");
  int err = insta::launch_norm_ratio(n, a, b, out, cuda_stream);
  if (err) return cuda_fail(err, "grad_norm_ratio");
  return INSTA_OK;
}

// ---------------------------------------------------------------------------
// INSTA-Size device steps
// ---------------------------------------------------------------------------
insta_status insta_stage_gradients(insta_graph* g, const float* d_arc_mean, float* stage_grad, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "stage_gradients: NULL graph");
  insta::DevGraph& d = g->d;
  if (d.e > 0 && (!d_arc_mean || !stage_grad)) return fail(INSTA_E_ARG, "stage_gradients: NULL array");
  if (d.e > 0 && !d.arc_class) return fail(INSTA_E_ARG, "stage_gradients: the graph has no arc_class");
  cudaSetDevice(d.device);
  int err = insta::launch_stage_gradients(d, d_arc_mean, stage_grad, cuda_stream);
  if (err) return cuda_fail(err, "stage_gradients");
  return INSTA_OK;
}

insta_status insta_select_stages(insta_graph* g, const float* stage_grad, float threshold, int32_t* out_arcs,
                                 int32_t* out_count, void* cuda_stream) {
  if (!g) return fail(INSTA_E_ARG, "select_stages: NULL graph");
  insta::DevGraph& d = g->d;
  if (!out_count || (d.e > 0 && (!stage_grad || !out_arcs))) return fail(INSTA_E_ARG, "select_stages: NULL array");
  if (!std::isfinite(threshold) || threshold < 0.f) return fail(INSTA_E_ARG, "select_stages: threshold must be >= 0");
  cudaSetDevice(d.device);
  int err = insta::launch_select_stages(d, stage_grad, threshold, out_arcs, out_count, cuda_stream);
  if (err) return cuda_fail(err, "select_stages");
  return INSTA_OK;
}

// debug builds (-DTK_STATS): merge batches of the Top-K kernel by survivor count (33 counters)
int insta_debug_topk_stats(unsigned long long* out) { return insta::topk_stats(out); }

insta_status insta_last_forward_stats(insta_graph* g, int64_t* pins_recomputed) {
  if (!g) return fail(INSTA_E_ARG, "stats: NULL graph");
  insta::DevGraph& d = g->d;
  if (pins_recomputed) {
    if (d.last_incremental) {
      unsigned long long c[2] = {0, 0};
      cudaError_t e = cudaMemcpy(c, d.counters, sizeof c, cudaMemcpyDeviceToHost);
      if (e != cudaSuccess) return cuda_fail(int(e), "stats");
      *pins_recomputed = int64_t(c[0]);
    } else {
      *pins_recomputed = d.last_recomputed;
    }
  }
  return INSTA_OK;
}

}  // extern "C"
