"""ctypes wrapper around liboracle.so -- the fp64 CPU oracle (TEST INFRASTRUCTURE).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(paper_conf_dac_lugklr25_b200) never does.

All functions take a ``synth.Graph``-like object (caller order, fp32 or fp64
arrays) and compute in fp64 (oracle/oracle.c).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liboracle.so")
_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")   # all-core build (bench cpu_baseline only)
_lib = None
_lib_omp = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    for out, extra in ((_LIB, []), (_LIB_OMP, ["-fopenmp"])):
        if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(src):
            subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fPIC", "-shared",
                                   "-Wall", *extra, "-o", out, src, "-lm"])
    return _LIB


def lib(omp: bool = False):
    """The serial oracle, or (omp=True) the OpenMP level-parallel build of the same source: forward
    identical, backward equal to rounding (atomic pushes), used only to time the all-core baseline."""
    global _lib, _lib_omp
    if omp:
        if _lib_omp is None:
            build()
            _lib_omp = ctypes.CDLL(_LIB_OMP)
        return _lib_omp
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
    return _lib


class _OrcGraph(ctypes.Structure):
    _fields_ = [
        ("num_pins", ctypes.c_int32),
        ("num_arcs", ctypes.c_int64),
        ("arc_from", ctypes.c_void_p),
        ("arc_to", ctypes.c_void_p),
        ("arc_unate", ctypes.c_void_p),
        ("arc_mean", ctypes.c_void_p),
        ("arc_sigma", ctypes.c_void_p),
        ("src_mean", ctypes.c_void_p),
        ("src_sigma", ctypes.c_void_p),
        ("num_endpoints", ctypes.c_int32),
        ("ep_pin", ctypes.c_void_p),
        ("ep_rat", ctypes.c_void_p),
    ]


def _p(a):
    return None if a is None else a.ctypes.data


class OracleError(RuntimeError):
    pass


def _check(st):
    if st == 1:
        raise OracleError("oracle: bad argument")
    if st == 2:
        raise OracleError("oracle: combinational cycle")
    if st:
        raise OracleError(f"oracle: status {st}")


class OGraph:
    """fp64 copies of a graph's arrays + the C struct pointing at them."""

    def __init__(self, g):
        self.N = int(g.num_pins)
        self.E = int(np.asarray(g.arc_from).shape[0])
        self.P = int(np.asarray(g.ep_pin).shape[0])
        self.arc_from = np.ascontiguousarray(g.arc_from, np.int32)
        self.arc_to = np.ascontiguousarray(g.arc_to, np.int32)
        self.arc_unate = np.ascontiguousarray(g.arc_unate, np.uint8)
        self.arc_mean = np.ascontiguousarray(np.asarray(g.arc_mean, np.float64).reshape(self.E, 2))
        self.arc_sigma = np.ascontiguousarray(np.asarray(g.arc_sigma, np.float64).reshape(self.E, 2))
        self.src_mean = None if g.src_mean is None else np.ascontiguousarray(np.asarray(g.src_mean, np.float64).reshape(self.N, 2))
        self.src_sigma = None if g.src_sigma is None else np.ascontiguousarray(np.asarray(g.src_sigma, np.float64).reshape(self.N, 2))
        self.ep_pin = np.ascontiguousarray(g.ep_pin, np.int32)
        self.ep_rat = np.ascontiguousarray(np.asarray(g.ep_rat, np.float64).reshape(self.P, 2))
        self.c = _OrcGraph(self.N, self.E, _p(self.arc_from), _p(self.arc_to), _p(self.arc_unate),
                           _p(self.arc_mean), _p(self.arc_sigma), _p(self.src_mean), _p(self.src_sigma),
                           self.P, _p(self.ep_pin), _p(self.ep_rat))


def _og(g):
    return g if isinstance(g, OGraph) else OGraph(g)


def levelize(num_pins, arc_from, arc_to):
    """Returns dict(level, order, fanin_ptr, fanin_arc, fanout_ptr, fanout_arc, num_levels)."""
    arc_from = np.ascontiguousarray(arc_from, np.int32)
    arc_to = np.ascontiguousarray(arc_to, np.int32)
    N, E = int(num_pins), int(arc_from.shape[0])
    out = dict(level=np.zeros(N, np.int32), order=np.zeros(N, np.int32),
               fanin_ptr=np.zeros(N + 1, np.int32), fanin_arc=np.zeros(E, np.int32),
               fanout_ptr=np.zeros(N + 1, np.int32), fanout_arc=np.zeros(E, np.int32))
    nl = ctypes.c_int32(0)
    L = lib()
    L.orc_levelize.argtypes = [ctypes.c_int32, ctypes.c_int64] + [ctypes.c_void_p] * 9
    _check(L.orc_levelize(N, E, _p(arc_from), _p(arc_to), _p(out["level"]), _p(out["order"]),
                          _p(out["fanin_ptr"]), _p(out["fanin_arc"]), _p(out["fanout_ptr"]),
                          _p(out["fanout_arc"]), ctypes.byref(nl)))
    out["num_levels"] = int(nl.value)
    return out


def forward(g, n_sigma=3.0, tau=0.0, omp=False):
    """Returns dict(A, sigma, mu [N,2], win_arc, win_s [N,2], gap [N,2])."""
    og = _og(g)
    N = og.N
    A = np.zeros((N, 2)); sig = np.zeros((N, 2)); mu = np.zeros((N, 2))
    wa = np.zeros((N, 2), np.int32); ws = np.zeros((N, 2), np.int8); gap = np.zeros((N, 2))
    L = lib(omp)
    L.orc_forward.argtypes = [ctypes.c_void_p, ctypes.c_double, ctypes.c_double] + [ctypes.c_void_p] * 6
    _check(L.orc_forward(ctypes.byref(og.c), float(n_sigma), float(tau), _p(A), _p(sig), _p(mu),
                         _p(wa), _p(ws), _p(gap)))
    return dict(A=A, sigma=sig, mu=mu, win_arc=wa, win_s=ws, gap=gap)


def slack(g, A):
    """Returns dict(slack [P], rf_star [P], wns, tns, num_viol)."""
    og = _og(g)
    A = np.ascontiguousarray(A, np.float64)
    s = np.zeros(og.P); r = np.zeros(og.P, np.uint8)
    wns = ctypes.c_double(); tns = ctypes.c_double(); nv = ctypes.c_int32()
    L = lib()
    L.orc_slack.argtypes = [ctypes.c_void_p] * 7
    _check(L.orc_slack(ctypes.byref(og.c), _p(A), _p(s), _p(r), ctypes.byref(wns), ctypes.byref(tns),
                       ctypes.byref(nv)))
    return dict(slack=s, rf_star=r, wns=wns.value, tns=tns.value, num_viol=nv.value)


def backward(g, n_sigma=3.0, tau=0.0, dslack=None, omp=False):
    """Returns dict(d_mean, d_sigma [E,2], d_src_mean, d_src_sigma, abar [N,2])."""
    og = _og(g)
    E, N = og.E, og.N
    dm = np.zeros((E, 2)); ds = np.zeros((E, 2))
    dsm = np.zeros((N, 2)); dss = np.zeros((N, 2)); ab = np.zeros((N, 2))
    if dslack is not None:
        dslack = np.ascontiguousarray(dslack, np.float64)
    L = lib(omp)
    L.orc_backward.argtypes = [ctypes.c_void_p, ctypes.c_double, ctypes.c_double] + [ctypes.c_void_p] * 6
    _check(L.orc_backward(ctypes.byref(og.c), float(n_sigma), float(tau), _p(dslack), _p(dm), _p(ds),
                          _p(dsm), _p(dss), _p(ab)))
    return dict(d_mean=dm, d_sigma=ds, d_src_mean=dsm, d_src_sigma=dss, abar=ab)


def tie_taint(g, n_sigma=3.0, eps=1e-3, margin=1.0):
    """Test support: (fwd_taint [N,2] bool, arc_taint [E,2] bool) for hard-mode parity."""
    og = _og(g)
    ft = np.zeros((og.N, 2), np.uint8); at = np.zeros((og.E, 2), np.uint8)
    L = lib()
    L.orc_tie_taint.argtypes = [ctypes.c_void_p, ctypes.c_double, ctypes.c_double, ctypes.c_double,
                                ctypes.c_void_p, ctypes.c_void_p]
    _check(L.orc_tie_taint(ctypes.byref(og.c), float(n_sigma), float(eps), float(margin), _p(ft), _p(at)))
    return ft.astype(bool), at.astype(bool)


def validate(g, n_sigma=3.0, tau=0.0) -> int:
    og = _og(g)
    L = lib()
    L.orc_validate.argtypes = [ctypes.c_void_p, ctypes.c_double, ctypes.c_double]
    return int(L.orc_validate(ctypes.byref(og.c), float(n_sigma), float(tau)))


def topk_forward(g, n_sigma=3.0, K=4):
    """NEXT 1, Alg 1 + Alg 2: Top-K unique-startpoint queues.
    Returns dict(A, mu, sigma [N,2,K] float64, sp [N,2,K] int32 caller ids, -1 = empty)."""
    og = _og(g)
    N = og.N
    A = np.zeros((N, 2, K)); mu = np.zeros((N, 2, K)); sig = np.zeros((N, 2, K))
    sp = np.zeros((N, 2, K), np.int32)
    L = lib()
    L.orc_topk_forward.argtypes = [ctypes.c_void_p, ctypes.c_double, ctypes.c_int32] + [ctypes.c_void_p] * 4
    _check(L.orc_topk_forward(ctypes.byref(og.c), float(n_sigma), int(K), _p(A), _p(mu), _p(sig), _p(sp)))
    return dict(A=A, mu=mu, sigma=sig, sp=sp)


def topk_taint(g, n_sigma=3.0, K=4, eps=1e-3):
    """Test support: [N,2] bool, queue rows whose startpoint SET may differ on another correct
    implementation (boundary near tie within eps, or an uncertain parent entry that can reach the row)."""
    og = _og(g)
    t = np.zeros((og.N, 2), np.uint8)
    L = lib()
    L.orc_topk_taint.argtypes = [ctypes.c_void_p, ctypes.c_double, ctypes.c_int32, ctypes.c_double, ctypes.c_void_p]
    _check(L.orc_topk_taint(ctypes.byref(og.c), float(n_sigma), int(K), float(eps), _p(t)))
    return t.astype(bool)


def topk_slack(g, q, rat_table=None):
    """CPPR slack over Top-K queues q (from topk_forward).  rat_table = (ptr [P+1], sp [M], rat [M,2]) or None.
    Returns dict(slack, rf_star, k_star, sp_star [P], wns, tns, num_viol)."""
    og = _og(g)
    K = int(q["A"].shape[2])
    A = np.ascontiguousarray(q["A"], np.float64)
    sp = np.ascontiguousarray(q["sp"], np.int32)
    rp = rs = rv = None
    if rat_table is not None:
        rp = np.ascontiguousarray(rat_table[0], np.int32)
        rs = np.ascontiguousarray(rat_table[1], np.int32)
        rv = np.ascontiguousarray(np.asarray(rat_table[2], np.float64).reshape(-1, 2))
    s = np.zeros(og.P); r = np.zeros(og.P, np.uint8); ks = np.zeros(og.P, np.int32); ss = np.zeros(og.P, np.int32)
    wns = ctypes.c_double(); tns = ctypes.c_double(); nv = ctypes.c_int32()
    L = lib()
    L.orc_topk_slack.argtypes = [ctypes.c_void_p, ctypes.c_int32] + [ctypes.c_void_p] * 12
    _check(L.orc_topk_slack(ctypes.byref(og.c), K, _p(A), _p(sp), _p(rp), _p(rs), _p(rv), _p(s), _p(r), _p(ks),
                            _p(ss), ctypes.byref(wns), ctypes.byref(tns), ctypes.byref(nv)))
    return dict(slack=s, rf_star=r, k_star=ks, sp_star=ss, wns=wns.value, tns=tns.value, num_viol=nv.value)


def clark_forward(g, n_sigma=3.0):
    """NEXT 2: Clark moment-matching merge.  Returns dict(A, mu, sigma [N,2])."""
    og = _og(g)
    N = og.N
    A = np.zeros((N, 2)); mu = np.zeros((N, 2)); sig = np.zeros((N, 2))
    L = lib()
    L.orc_clark_forward.argtypes = [ctypes.c_void_p, ctypes.c_double] + [ctypes.c_void_p] * 3
    _check(L.orc_clark_forward(ctypes.byref(og.c), float(n_sigma), _p(A), _p(mu), _p(sig)))
    return dict(A=A, mu=mu, sigma=sig)


def clark_backward(g, n_sigma=3.0, dslack=None):
    """Backward of the Clark path.  Returns dict(d_mean, d_sigma [E,2], d_src_mean, d_src_sigma [N,2])."""
    og = _og(g)
    E, N = og.E, og.N
    dm = np.zeros((E, 2)); ds = np.zeros((E, 2)); dsm = np.zeros((N, 2)); dss = np.zeros((N, 2))
    if dslack is not None:
        dslack = np.ascontiguousarray(dslack, np.float64)
    L = lib()
    L.orc_clark_backward.argtypes = [ctypes.c_void_p, ctypes.c_double] + [ctypes.c_void_p] * 5
    _check(L.orc_clark_backward(ctypes.byref(og.c), float(n_sigma), _p(dslack), _p(dm), _p(ds), _p(dsm), _p(dss)))
    return dict(d_mean=dm, d_sigma=ds, d_src_mean=dsm, d_src_sigma=dss)


def timing_loss(g, x, y, w, lambda_rc=1.0):
    """NEXT 4, Eq 7: returns (L, grad_x [N], grad_y [N])."""
    og = _og(g)
    x = np.ascontiguousarray(x, np.float64); y = np.ascontiguousarray(y, np.float64)
    w = np.ascontiguousarray(w, np.float64)
    gx = np.zeros(og.N); gy = np.zeros(og.N); L = ctypes.c_double()
    lb = lib()
    lb.orc_timing_loss.argtypes = [ctypes.c_void_p] * 4 + [ctypes.c_double] + [ctypes.c_void_p] * 3
    _check(lb.orc_timing_loss(ctypes.byref(og.c), _p(x), _p(y), _p(w), float(lambda_rc), ctypes.byref(L), _p(gx),
                              _p(gy)))
    return L.value, gx, gy


def stage_gradients(g, d_mean):
    """NEXT 3 (R22): per cell arc, the gradient sum of the cell arc and its driving net arc; 0 for net arcs."""
    og = _og(g)
    cls = np.ascontiguousarray(g.arc_class, np.uint8)
    dm = np.ascontiguousarray(np.asarray(d_mean, np.float64).reshape(og.E, 2))
    out = np.zeros(og.E)
    L = lib()
    L.orc_stage_gradients.argtypes = [ctypes.c_void_p] * 4
    _check(L.orc_stage_gradients(ctypes.byref(og.c), _p(cls), _p(dm), _p(out)))
    return out
