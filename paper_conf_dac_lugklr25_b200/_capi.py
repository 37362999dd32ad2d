"""ctypes declarations of include/insta.h (argument marshalling only).

Loading fails loudly if libinsta.so is missing: there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libinsta.so")

c_i32p = ctypes.POINTER(ctypes.c_int32)
c_vp = ctypes.c_void_p


class insta_graph_desc(ctypes.Structure):
    _fields_ = [
        ("num_pins", ctypes.c_int32),
        ("num_arcs", ctypes.c_int64),
        ("arc_from", c_vp),
        ("arc_to", c_vp),
        ("arc_unate", c_vp),
        ("arc_mean", c_vp),
        ("arc_sigma", c_vp),
        ("src_mean", c_vp),
        ("src_sigma", c_vp),
        ("num_endpoints", ctypes.c_int32),
        ("ep_pin", c_vp),
        ("ep_rat", c_vp),
        ("arc_class", c_vp),
        ("device", ctypes.c_int32),
    ]


class insta_opts(ctypes.Structure):
    _fields_ = [("n_sigma", ctypes.c_float), ("tau", ctypes.c_float),
                ("want_grad_sigma", ctypes.c_int32), ("schedule", ctypes.c_int32), ("cone_max", ctypes.c_int64)]


class insta_summary(ctypes.Structure):
    _fields_ = [("wns", ctypes.c_double), ("tns", ctypes.c_double),
                ("num_violations", ctypes.c_int32), ("num_levels", ctypes.c_int32)]


class insta_scenario(ctypes.Structure):
    _fields_ = [("n_sigma", ctypes.c_float), ("derate_cell", ctypes.c_float), ("derate_net", ctypes.c_float),
                ("n_delta", ctypes.c_int32), ("delta_arc", c_vp), ("delta_mean", c_vp), ("delta_sigma", c_vp)]


class insta_schedule(ctypes.Structure):
    _fields_ = [("num_heads", ctypes.c_int32), ("num_super_levels", ctypes.c_int32),
                ("num_entries", ctypes.c_int64), ("num_folded", ctypes.c_int64),
                ("num_light_fanout", ctypes.c_int64), ("fwd_steps", ctypes.c_int32), ("bwd_steps", ctypes.c_int32)]


# name -> (restype, argtypes); every symbol declared in include/insta.h
SIGNATURES = {
    "insta_levelize": (ctypes.c_int, [ctypes.c_int32, ctypes.c_int64, c_vp, c_vp, c_vp, c_vp, c_vp, c_vp,
                                      c_vp, c_vp, c_vp]),
    "insta_graph_create": (ctypes.c_int, [ctypes.POINTER(insta_graph_desc), ctypes.POINTER(c_vp)]),
    "insta_graph_destroy": (None, [c_vp]),
    "insta_graph_export": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_graph_sizes": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_graph_schedule": (ctypes.c_int, [c_vp, ctypes.POINTER(insta_schedule)]),
    "insta_forward": (ctypes.c_int, [c_vp, ctypes.POINTER(insta_opts), c_vp, ctypes.POINTER(insta_summary)]),
    "insta_slack": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, ctypes.POINTER(insta_summary)]),
    "insta_arrivals": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_backward": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_update_arcs": (ctypes.c_int, [c_vp, ctypes.c_int64, c_vp, c_vp, c_vp, ctypes.c_int32, c_vp]),
    "insta_last_forward_stats": (ctypes.c_int, [c_vp, c_vp]),
    "insta_backward_update": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp]),
    "insta_last_backward_stats": (ctypes.c_int, [c_vp, c_vp]),
    "insta_forward_batch": (ctypes.c_int, [c_vp, ctypes.c_int32, ctypes.POINTER(insta_scenario), ctypes.c_float,
                                           c_vp, c_vp, c_vp]),
    "insta_eval_candidates": (ctypes.c_int, [c_vp, ctypes.c_int32, c_vp, c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_set_cppr_rat": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp]),
    "insta_topk_forward": (ctypes.c_int, [c_vp, ctypes.c_int32, ctypes.c_float, c_vp]),
    "insta_topk_slack": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, ctypes.POINTER(insta_summary)]),
    "insta_topk_critical": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp]),
    "insta_topk_queues": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_clark_forward": (ctypes.c_int, [c_vp, ctypes.c_float, c_vp, ctypes.POINTER(insta_summary)]),
    "insta_clark_results": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_clark_backward": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, c_vp, c_vp]),
    "insta_stage_gradients": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp]),
    "insta_select_stages": (ctypes.c_int, [c_vp, c_vp, ctypes.c_float, c_vp, c_vp, c_vp]),
    "insta_timing_loss": (ctypes.c_int, [c_vp, c_vp, c_vp, c_vp, ctypes.c_float, c_vp, c_vp, c_vp, c_vp]),
    "insta_grad_norm_ratio": (ctypes.c_int, [ctypes.c_int64, c_vp, c_vp, c_vp, c_vp]),
    "insta_debug_topk_stats": (ctypes.c_int, [c_vp]),
    "insta_last_error": (ctypes.c_char_p, []),
    "insta_version": (ctypes.c_char_p, []),
}

STATUS = {0: "OK", 1: "E_ARG", 2: "E_CYCLE", 3: "E_CUDA", 4: "E_NOMEM", 5: "E_STATE"}

_lib = None


def load():
    """Load libinsta.so (building it first if the sources are newer)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        try:
            from . import build as _b
            _b.build()
        except Exception as e:  # pragma: no cover - fail loudly, never fall back
            raise ImportError(f"libinsta.so is missing and could not be built: {e}") from e
    lib = ctypes.CDLL(LIB_PATH)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib


class InstaError(RuntimeError):
    def __init__(self, status: int, where: str):
        msg = load().insta_last_error().decode(errors="replace")
        super().__init__(f"{where}: {STATUS.get(status, status)}: {msg}")
        self.status = status


def check(status: int, where: str):
    if status != 0:
        raise InstaError(status, where)
