"""B200-native INSTA hot path: Python binding over the C ABI (include/insta.h).

Argument marshalling only -- every step of the path runs in libinsta.so's
CUDA kernels.  torch supplies device memory and streams.

    g = Graph(desc)                      # validate + levelize + upload
    s = g.forward(n_sigma=3.0, tau=0.0)  # arrivals -> slack -> WNS/TNS
    d_mean = g.backward()                # dTNS/d(arc mean), caller arc order
"""
from __future__ import annotations

import ctypes
import dataclasses

import numpy as np

from . import _capi
from ._capi import InstaError, check

__all__ = ["Graph", "Summary", "InstaError", "levelize", "version", "grad_norm_ratio"]


@dataclasses.dataclass
class Summary:
    wns: float
    tns: float
    num_violations: int
    num_levels: int


def version() -> str:
    return _capi.load().insta_version().decode()


def _np(a, dtype, shape=None):
    a = np.ascontiguousarray(a, dtype=dtype)
    if shape is not None:
        a = a.reshape(shape)
    return a


def _ptr(a):
    return None if a is None else a.ctypes.data


def levelize(num_pins: int, arc_from, arc_to) -> dict:
    """Host-only levelization through the C ABI (insta_levelize)."""
    lib = _capi.load()
    af = _np(arc_from, np.int32)
    at = _np(arc_to, np.int32)
    N, E = int(num_pins), int(af.shape[0])
    out = dict(level=np.zeros(N, np.int32), order=np.zeros(N, np.int32),
               fanin_ptr=np.zeros(N + 1, np.int32), fanin_arc=np.zeros(E, np.int32),
               fanout_ptr=np.zeros(N + 1, np.int32), fanout_arc=np.zeros(E, np.int32))
    nl = ctypes.c_int32(0)
    check(lib.insta_levelize(N, E, _ptr(af), _ptr(at), _ptr(out["level"]), _ptr(out["order"]),
                             _ptr(out["fanin_ptr"]), _ptr(out["fanin_arc"]), _ptr(out["fanout_ptr"]),
                             _ptr(out["fanout_arc"]), ctypes.byref(nl)), "insta_levelize")
    out["num_levels"] = int(nl.value)
    return out


def grad_norm_ratio(a, b, stream=None):
    """insta_grad_norm_ratio (Eq 8): ||a|| / ||b|| of two float32 device tensors, as a float64 device scalar."""
    import torch
    a = a.contiguous().float()
    b = b.contiguous().float()
    if a.numel() != b.numel():   # the ABI reads n elements of both
        raise ValueError(f"grad_norm_ratio: a has {a.numel()} elements, b has {b.numel()}")
    out = torch.empty(1, dtype=torch.float64, device=a.device)
    st = ctypes.c_void_p((stream or torch.cuda.current_stream(a.device)).cuda_stream)
    check(_capi.load().insta_grad_norm_ratio(int(a.numel()), _dptr(a), _dptr(b), _dptr(out), st),
          "insta_grad_norm_ratio")
    return out


def _stream(torch, device):
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


def _dptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


class Graph:
    """A timing graph resident on one GPU (opaque insta_graph)."""

    def __init__(self, g, device: int = 0):
        import torch  # plumbing only: device memory + streams
        self._torch = torch
        self.lib = _capi.load()
        self.device = torch.device("cuda", device)
        self.num_pins = int(g.num_pins)
        self._arrs = dict(
            arc_from=_np(g.arc_from, np.int32), arc_to=_np(g.arc_to, np.int32),
            arc_unate=_np(g.arc_unate, np.uint8),
            arc_mean=_np(g.arc_mean, np.float32), arc_sigma=_np(g.arc_sigma, np.float32),
            src_mean=None if getattr(g, "src_mean", None) is None else _np(g.src_mean, np.float32),
            src_sigma=None if getattr(g, "src_sigma", None) is None else _np(g.src_sigma, np.float32),
            ep_pin=_np(g.ep_pin, np.int32), ep_rat=_np(g.ep_rat, np.float32),
            arc_class=None if getattr(g, "arc_class", None) is None else _np(g.arc_class, np.uint8))
        a = self._arrs
        self.num_arcs = int(a["arc_from"].shape[0])
        self.num_endpoints = int(a["ep_pin"].shape[0])
        desc = _capi.insta_graph_desc(
            self.num_pins, self.num_arcs, _ptr(a["arc_from"]), _ptr(a["arc_to"]), _ptr(a["arc_unate"]),
            _ptr(a["arc_mean"]), _ptr(a["arc_sigma"]), _ptr(a["src_mean"]), _ptr(a["src_sigma"]),
            self.num_endpoints, _ptr(a["ep_pin"]), _ptr(a["ep_rat"]), _ptr(a["arc_class"]), int(device))
        h = ctypes.c_void_p()
        check(self.lib.insta_graph_create(ctypes.byref(desc), ctypes.byref(h)), "insta_graph_create")
        self._h = h
        self._arrs = None   # the library copied everything
        nl = ctypes.c_int32()
        check(self.lib.insta_graph_sizes(self._h, None, None, None, ctypes.byref(nl)), "insta_graph_sizes")
        self.num_levels = int(nl.value)

    def schedule(self) -> dict:
        """insta_graph_schedule: the stage-folded schedule of the persistent passes."""
        sc = _capi.insta_schedule()
        check(self.lib.insta_graph_schedule(self._h, ctypes.byref(sc)), "insta_graph_schedule")
        return {name: int(getattr(sc, name)) for name, _ in sc._fields_}

    # ------------------------------------------------------------------ lifetime
    def close(self):
        if getattr(self, "_h", None):
            self.lib.insta_graph_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # ------------------------------------------------------------------ calls
    def _st(self, stream=None):
        if stream is not None:
            return ctypes.c_void_p(stream.cuda_stream)
        return _stream(self._torch, self.device)

    def _dev(self, x, dtype, stream=None):
        """A contiguous device copy of x allocated on the call's stream (the caching allocator then
        never hands its memory to another stream while the library kernel still reads it)."""
        t = self._torch
        with t.cuda.stream(stream or t.cuda.current_stream(self.device)):
            return t.as_tensor(x, dtype=dtype, device=self.device).contiguous()

    def forward(self, n_sigma: float = 3.0, tau: float = 0.0, schedule: int = 0, sync: bool = True,
                stream=None, cone_max: int = 0):
        """insta_forward: arrivals -> endpoint slack -> WNS/TNS.  Returns a Summary if sync.
        cone_max: incremental policy (include/insta.h): 0 default, < 0 never, > 0 max arcs for the cone pass."""
        opts = _capi.insta_opts(float(n_sigma), float(tau), 0, int(schedule), int(cone_max))
        out = _capi.insta_summary() if sync else None
        check(self.lib.insta_forward(self._h, ctypes.byref(opts), self._st(stream),
                                     ctypes.byref(out) if out is not None else None), "insta_forward")
        if out is None:
            return None
        return Summary(out.wns, out.tns, out.num_violations, out.num_levels)

    def slack(self, stream=None):
        """insta_slack: (slack float32[P], rf_star uint8[P]) device tensors, caller endpoint order."""
        t = self._torch
        s = t.empty(self.num_endpoints, dtype=t.float32, device=self.device)
        r = t.empty(self.num_endpoints, dtype=t.uint8, device=self.device)
        check(self.lib.insta_slack(self._h, _dptr(s), _dptr(r), self._st(stream), None), "insta_slack")
        return s, r

    def summary(self, stream=None) -> Summary:
        out = _capi.insta_summary()
        check(self.lib.insta_slack(self._h, None, None, self._st(stream), ctypes.byref(out)), "insta_slack")
        return Summary(out.wns, out.tns, out.num_violations, out.num_levels)

    def arrivals(self, stream=None):
        """insta_arrivals: (A, mean, sigma) float32[N,2] device tensors in caller pin order."""
        t = self._torch
        A, m, s = (t.empty((self.num_pins, 2), dtype=t.float32, device=self.device) for _ in range(3))
        check(self.lib.insta_arrivals(self._h, _dptr(A), _dptr(m), _dptr(s), self._st(stream)), "insta_arrivals")
        return A, m, s

    def backward(self, ep_seed=None, want_src: bool = False, out=None, stream=None, want_sigma: bool = False):
        """insta_backward: dL/d(arc mean) float32[E,2] (caller arc order); L = TNS if ep_seed is None.
        want_sigma: also dL/d(arc sigma) float32[E,2]; want_src: dL/d(src mean) float32[N,2].
        Returns d_mean, or a tuple (d_mean[, d_sigma][, d_src])."""
        t = self._torch
        d_mean = out if out is not None else t.empty((self.num_arcs, 2), dtype=t.float32, device=self.device)
        d_sig = t.empty((self.num_arcs, 2), dtype=t.float32, device=self.device) if want_sigma else None
        d_src = t.empty((self.num_pins, 2), dtype=t.float32, device=self.device) if want_src else None
        seed = None
        if ep_seed is not None:
            with t.cuda.stream(stream or t.cuda.current_stream(self.device)):   # allocated on the call's stream
                seed = t.as_tensor(ep_seed, dtype=t.float32, device=self.device).contiguous()
            if seed.numel() != self.num_endpoints:
                raise ValueError(f"ep_seed: expected {self.num_endpoints} values, got {seed.numel()}")
        check(self.lib.insta_backward(self._h, _dptr(seed), _dptr(d_mean), _dptr(d_sig), _dptr(d_src),
                                      self._st(stream)), "insta_backward")
        outs = (d_mean,) + ((d_sig,) if want_sigma else ()) + ((d_src,) if want_src else ())
        return outs if len(outs) > 1 else d_mean

    def backward_update(self, out, stream=None) -> bool:
        """insta_backward_update: the TNS gradient in `out` (float32[E,2] device tensor holding the
        previous call's result) brought up to date after incremental forwards, in the reverse cone
        of the change; the first call (or one after a full forward) runs the full backward.
        Returns True if the update ran incrementally."""
        inc = ctypes.c_int32(0)
        check(self.lib.insta_backward_update(self._h, _dptr(out), self._st(stream), ctypes.byref(inc)),
              "insta_backward_update")
        return bool(inc.value)

    def last_backward_stats(self) -> int:
        v = ctypes.c_int64()
        check(self.lib.insta_last_backward_stats(self._h, ctypes.byref(v)), "insta_last_backward_stats")
        return int(v.value)

    def update_arcs(self, arc_ids, mean, sigma, incremental: bool = True, stream=None):
        """insta_update_arcs: re-annotate arcs (device or host arrays; copied to the device)."""
        t = self._torch
        # temporaries live on the stream the library call is ordered on (the caching allocator
        # cannot hand their memory to another stream while the kernel still reads it)
        with t.cuda.stream(stream or t.cuda.current_stream(self.device)):
            ids = None if arc_ids is None else t.as_tensor(arc_ids, dtype=t.int32, device=self.device).contiguous()
            m = t.as_tensor(mean, dtype=t.float32, device=self.device).contiguous()
            s = t.as_tensor(sigma, dtype=t.float32, device=self.device).contiguous()
        n = self.num_arcs if ids is None else int(ids.numel())   # arc_ids None: every arc, caller order
        if m.numel() != 2 * n or s.numel() != 2 * n:
            raise ValueError(f"update_arcs: mean and sigma need {2 * n} values ([n][2]), got {m.numel()}, {s.numel()}")
        check(self.lib.insta_update_arcs(self._h, n, _dptr(ids), _dptr(m), _dptr(s),
                                         int(bool(incremental)), self._st(stream)), "insta_update_arcs")

    # ------------------------------------------------------------------ Top-K / CPPR
    def set_cppr_rat(self, rat_ptr=None, rat_sp=None, rat=None):
        """insta_set_cppr_rat: per-(endpoint, startpoint) required times (host arrays; None clears)."""
        if rat_ptr is None:
            check(self.lib.insta_set_cppr_rat(self._h, None, None, None), "insta_set_cppr_rat")
            return
        rp = _np(rat_ptr, np.int32)
        rs = _np(rat_sp, np.int32)
        rv = _np(rat, np.float32, (-1, 2))
        check(self.lib.insta_set_cppr_rat(self._h, _ptr(rp), _ptr(rs), _ptr(rv)), "insta_set_cppr_rat")

    def topk_forward(self, K: int, n_sigma: float = 3.0, stream=None):
        """insta_topk_forward: Top-K unique-startpoint queues (Alg 1 + Alg 2)."""
        self.topk_K = int(K)
        check(self.lib.insta_topk_forward(self._h, int(K), float(n_sigma), self._st(stream)), "insta_topk_forward")

    def topk_slack(self, stream=None, sync: bool = True):
        """insta_topk_slack: CPPR slack.  Returns (Summary or None, slack float32[P], sp_star int32[P])."""
        t = self._torch
        s = t.empty(self.num_endpoints, dtype=t.float32, device=self.device)
        sp = t.empty(self.num_endpoints, dtype=t.int32, device=self.device)
        out = _capi.insta_summary() if sync else None
        check(self.lib.insta_topk_slack(self._h, _dptr(s), _dptr(sp), self._st(stream),
                                        ctypes.byref(out) if out is not None else None), "insta_topk_slack")
        summ = None if out is None else Summary(out.wns, out.tns, out.num_violations, out.num_levels)
        return summ, s, sp

    def topk_critical(self, stream=None):
        """insta_topk_critical: (rf_star uint8[P], k_star int32[P]) of the last topk_slack."""
        t = self._torch
        r = t.empty(self.num_endpoints, dtype=t.uint8, device=self.device)
        k = t.empty(self.num_endpoints, dtype=t.int32, device=self.device)
        check(self.lib.insta_topk_critical(self._h, _dptr(r), _dptr(k), self._st(stream)), "insta_topk_critical")
        return r, k

    def topk_queues(self, stream=None):
        """insta_topk_queues: dict(A, mean, sigma float32[N,2,K], sp int32[N,2,K]) in caller pin order."""
        t = self._torch
        K = self.topk_K
        A, m, s = (t.empty((self.num_pins, 2, K), dtype=t.float32, device=self.device) for _ in range(3))
        sp = t.empty((self.num_pins, 2, K), dtype=t.int32, device=self.device)
        check(self.lib.insta_topk_queues(self._h, _dptr(A), _dptr(m), _dptr(s), _dptr(sp), self._st(stream)),
              "insta_topk_queues")
        return dict(A=A, mean=m, sigma=s, sp=sp)

    # ------------------------------------------------------------------ Clark merge
    def clark_forward(self, n_sigma: float = 3.0, sync: bool = True, stream=None):
        """insta_clark_forward: Clark moment-matching propagation + slack.  Returns a Summary if sync."""
        out = _capi.insta_summary() if sync else None
        check(self.lib.insta_clark_forward(self._h, float(n_sigma), self._st(stream),
                                           ctypes.byref(out) if out is not None else None), "insta_clark_forward")
        return None if out is None else Summary(out.wns, out.tns, out.num_violations, out.num_levels)

    def clark_results(self, stream=None):
        """insta_clark_results: dict(A, mean, sigma float32[N,2], slack float32[P], rf_star uint8[P])."""
        t = self._torch
        A, m, s = (t.empty((self.num_pins, 2), dtype=t.float32, device=self.device) for _ in range(3))
        sl = t.empty(self.num_endpoints, dtype=t.float32, device=self.device)
        rf = t.empty(self.num_endpoints, dtype=t.uint8, device=self.device)
        check(self.lib.insta_clark_results(self._h, _dptr(A), _dptr(m), _dptr(s), _dptr(sl), _dptr(rf),
                                           self._st(stream)), "insta_clark_results")
        return dict(A=A, mean=m, sigma=s, slack=sl, rf_star=rf)

    def clark_backward(self, ep_seed=None, want_sigma: bool = False, want_src: bool = False, stream=None):
        """insta_clark_backward: d_mean float32[E,2] (+ d_sigma [E,2], + d_src [N,2]) of L = TNS or sum seed*slack."""
        t = self._torch
        d_mean = t.empty((self.num_arcs, 2), dtype=t.float32, device=self.device)
        d_sig = t.empty((self.num_arcs, 2), dtype=t.float32, device=self.device) if want_sigma else None
        d_src = t.empty((self.num_pins, 2), dtype=t.float32, device=self.device) if want_src else None
        seed = None if ep_seed is None else self._dev(ep_seed, t.float32, stream)
        check(self.lib.insta_clark_backward(self._h, _dptr(seed), _dptr(d_mean), _dptr(d_sig), _dptr(d_src),
                                            self._st(stream)), "insta_clark_backward")
        outs = (d_mean,) + ((d_sig,) if want_sigma else ()) + ((d_src,) if want_src else ())
        return outs if len(outs) > 1 else d_mean

    # ------------------------------------------------------------------ INSTA-Size steps
    def stage_gradients(self, d_mean, stream=None):
        """insta_stage_gradients: float32[E] stage gradient per cell arc (0 for net arcs)."""
        t = self._torch
        dm = self._dev(d_mean, t.float32, stream)
        out = t.empty(self.num_arcs, dtype=t.float32, device=self.device)
        check(self.lib.insta_stage_gradients(self._h, _dptr(dm), _dptr(out), self._st(stream)), "insta_stage_gradients")
        return out

    def select_stages(self, stage_grad, threshold: float = 0.0, stream=None):
        """insta_select_stages: int32 device tensor of cell arc ids with grad < -threshold, most negative first."""
        t = self._torch
        arcs = t.empty(max(self.num_arcs, 1), dtype=t.int32, device=self.device)
        cnt = t.zeros(1, dtype=t.int32, device=self.device)
        check(self.lib.insta_select_stages(self._h, _dptr(stage_grad), float(threshold), _dptr(arcs), _dptr(cnt),
                                           self._st(stream)), "insta_select_stages")
        return arcs[: int(cnt.item())]

    # ------------------------------------------------------------------ INSTA-Place Eq 7
    def timing_loss(self, pin_x, pin_y, arc_w, lambda_rc: float = 1.0, want_grad: bool = True, stream=None):
        """insta_timing_loss: (L float64 device scalar, grad_x float32[N], grad_y float32[N]) of Eq 7."""
        t = self._torch
        x = self._dev(pin_x, t.float32, stream)
        y = self._dev(pin_y, t.float32, stream)
        w = self._dev(arc_w, t.float32, stream)
        L = t.empty(1, dtype=t.float64, device=self.device)
        gx = t.empty(self.num_pins, dtype=t.float32, device=self.device) if want_grad else None
        gy = t.empty(self.num_pins, dtype=t.float32, device=self.device) if want_grad else None
        check(self.lib.insta_timing_loss(self._h, _dptr(x), _dptr(y), _dptr(w), float(lambda_rc), _dptr(L), _dptr(gx),
                                         _dptr(gy), self._st(stream)), "insta_timing_loss")
        return L, gx, gy

    def forward_batch(self, scenarios, tau: float = 0.0, want_grad: bool = False, summaries=None, d_mean_sum=None,
                      stream=None):
        """insta_forward_batch: evaluate independent scenarios (dicts with n_sigma, derate_cell, derate_net and
        optional delta_arc / delta_mean / delta_sigma host arrays).  Returns (summaries float64[B,3] {wns, tns,
        num_violations} device tensor, d_mean_sum float32[E,2] or None)."""
        t = self._torch
        B = len(scenarios)
        arr = (_capi.insta_scenario * max(B, 1))()
        keep = []
        for k, sc in enumerate(scenarios):
            da = sc.get("delta_arc")
            n = 0 if da is None else len(da)
            if n:
                ids = _np(da, np.int32)
                dm = _np(sc["delta_mean"], np.float32, (n, 2))
                ds = _np(sc["delta_sigma"], np.float32, (n, 2))
                keep += [ids, dm, ds]
                arr[k] = _capi.insta_scenario(float(sc.get("n_sigma", 3.0)), float(sc.get("derate_cell", 1.0)),
                                              float(sc.get("derate_net", 1.0)), n, _ptr(ids), _ptr(dm), _ptr(ds))
            else:
                arr[k] = _capi.insta_scenario(float(sc.get("n_sigma", 3.0)), float(sc.get("derate_cell", 1.0)),
                                              float(sc.get("derate_net", 1.0)), 0, None, None, None)
        summ = summaries if summaries is not None else t.empty((B, 3), dtype=t.float64, device=self.device)
        dsum = None
        if want_grad:
            dsum = d_mean_sum if d_mean_sum is not None else t.empty((self.num_arcs, 2), dtype=t.float32,
                                                                      device=self.device)
        check(self.lib.insta_forward_batch(self._h, B, arr, float(tau), _dptr(summ), _dptr(dsum), self._st(stream)),
              "insta_forward_batch")
        return summ, dsum

    def eval_candidates(self, candidates, stream=None, summaries=None):
        """insta_eval_candidates: what-if summaries of sparse re-annotations (dicts with delta_arc /
        delta_mean / delta_sigma host arrays, e.g. synth.sizing_scenario), each applied, evaluated with the
        cone pass and reverted.  Returns float64[n, 3] {wns, tns, num_violations} device tensor."""
        return self.eval_packed(self.pack_candidates(candidates, stream), stream=stream, summaries=summaries)

    def eval_packed(self, packed, stream=None, summaries=None):
        """insta_eval_candidates on candidates already packed by pack_candidates (no host work per call)."""
        t = self._torch
        ptr, di, dm, ds = packed
        n = len(ptr) - 1
        out = summaries if summaries is not None else t.empty((n, 3), dtype=t.float64, device=self.device)
        check(self.lib.insta_eval_candidates(self._h, n, _ptr(ptr), _dptr(di), _dptr(dm), _dptr(ds), _dptr(out),
                                             self._st(stream)), "insta_eval_candidates")
        return out

    def pack_candidates(self, candidates, stream=None):
        """(cand_ptr host int32[n + 1], arc ids, mean, sigma device tensors) for eval_packed."""
        t = self._torch
        n = len(candidates)
        ptr = np.zeros(n + 1, np.int32)
        for k, c in enumerate(candidates):
            ptr[k + 1] = ptr[k] + len(c["delta_arc"])
        ids = np.concatenate([np.asarray(c["delta_arc"], np.int32) for c in candidates]) if n else np.zeros(0, np.int32)
        m = np.concatenate([np.asarray(c["delta_mean"], np.float32).reshape(-1, 2) for c in candidates]) if n else \
            np.zeros((0, 2), np.float32)
        sg = np.concatenate([np.asarray(c["delta_sigma"], np.float32).reshape(-1, 2) for c in candidates]) if n else \
            np.zeros((0, 2), np.float32)
        if len(ids) and (int(ids.min()) < 0 or int(ids.max()) >= self.num_arcs):   # the ABI reads them unchecked
            raise ValueError(f"eval_candidates: arc ids must be in [0, {self.num_arcs})")
        if len(m) != len(ids) or len(sg) != len(ids):
            raise ValueError("eval_candidates: delta_mean / delta_sigma need one [2] row per delta_arc")
        di, dm, ds = (self._dev(x, dt, stream) for x, dt in ((ids, t.int32), (m, t.float32), (sg, t.float32)))
        return ptr, di, dm, ds

    def last_forward_stats(self) -> int:
        v = ctypes.c_int64()
        check(self.lib.insta_last_forward_stats(self._h, ctypes.byref(v)), "insta_last_forward_stats")
        return int(v.value)

    def export(self) -> dict:
        """insta_graph_export: the levelization (host numpy) for bit-exact checks."""
        N, E = self.num_pins, self.num_arcs
        out = dict(level=np.zeros(N, np.int32), order=np.zeros(N, np.int32),
                   fanin_ptr=np.zeros(N + 1, np.int32), fanin_arc=np.zeros(E, np.int32),
                   fanout_ptr=np.zeros(N + 1, np.int32), fanout_arc=np.zeros(E, np.int32))
        check(self.lib.insta_graph_export(self._h, _ptr(out["level"]), _ptr(out["order"]), _ptr(out["fanin_ptr"]),
                                          _ptr(out["fanin_arc"]), _ptr(out["fanout_ptr"]), _ptr(out["fanout_arc"])),
              "insta_graph_export")
        out["num_levels"] = self.num_levels
        return out
