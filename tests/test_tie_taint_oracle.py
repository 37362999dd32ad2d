"""Pins of the oracle's near-tie taint (oracle/oracle.c orc_tie_taint), which
decides the hard-mode elements the GPU parity tests exempt (T2).

Planted exact ties on hand-built sigma = 0 DAGs: the taint must flag exactly
the tied merge and what it feeds (forward), and exactly the arcs the adjoint
of a violating endpoint may take through the tie (backward) -- nothing else.
A mask that is too broad would hide real GPU mismatches, one that is too
narrow would fail correct ones.
"""
import types

import numpy as np

import oracle

NS = 3.0


def graph(n, arcs, ep, rat, src_mean=None):
    """arcs: list of (from, to, mean) with mean equal for R and F, POS, sigma 0.  Startpoints
    arrive at (R, F) = (0, 0.5): every fall arrival is 0.5 ps later, so no endpoint has an
    rf tie (which would make its seed ambiguous, a taint source of its own)."""
    af = np.array([a for a, _, _ in arcs], np.int32)
    at = np.array([b for _, b, _ in arcs], np.int32)
    m = np.array([[x, x] for _, _, x in arcs], np.float32)
    sm = np.tile(np.array([0.0, 0.5], np.float32), (n, 1)) if src_mean is None else np.asarray(src_mean, np.float32)
    return types.SimpleNamespace(
        num_pins=n, arc_from=af, arc_to=at, arc_unate=np.zeros(len(arcs), np.uint8), arc_class=None,
        arc_mean=m, arc_sigma=np.zeros_like(m), src_mean=sm, src_sigma=np.zeros((n, 2), np.float32),
        ep_pin=np.array(ep, np.int32), ep_rat=np.array([[r, r] for r in rat], np.float32))


# pins: s=0, a=1, b=2, y=3, z=4 (endpoint), w=5 (endpoint on an untied branch), c=6
ARCS = [(0, 1, 5.0), (0, 2, 5.0), (1, 3, 1.0), (2, 3, 1.0), (3, 4, 2.0), (0, 6, 3.0), (6, 5, 1.0)]


def test_exact_tie_taints_its_cone_only():
    g = graph(7, ARCS, ep=[4, 5], rat=[0.0, 100.0])   # z violates (A = 8 > 0), w does not
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    want_f = np.zeros((7, 2), bool)
    want_f[[3, 4]] = True                               # the tied merge y and its sink z
    assert np.array_equal(ft, want_f)
    want_a = np.zeros((len(ARCS), 2), bool)
    want_a[[0, 1, 2, 3, 4], 1] = True                    # every arc the violating z's adjoint may take (rf* = F)
    assert np.array_equal(at, want_a)


def test_tie_without_adjoint_flow_taints_no_arc():
    g = graph(7, ARCS, ep=[4, 5], rat=[100.0, 100.0])   # no violation, slack far from 0
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    assert ft[[3, 4]].all() and not ft[[0, 1, 2, 5, 6]].any()
    assert not at.any()


def test_gap_above_eps_is_not_a_tie():
    arcs = list(ARCS)
    arcs[3] = (2, 3, 1.0 - 0.0625)                      # b's candidate 0.0625 ps below a's (> eps, > margin)
    g = graph(7, arcs, ep=[4, 5], rat=[0.0, 100.0])
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    assert not ft.any() and not at.any()


def test_near_tie_within_eps():
    arcs = list(ARCS)
    arcs[3] = (2, 3, 1.0 - 2.0 ** -12)                  # 0.00024 ps < eps = 1e-3: a near tie
    g = graph(7, arcs, ep=[4, 5], rat=[0.0, 100.0])
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    assert ft[[3, 4]].all() and not ft[[0, 1, 2, 5, 6]].any()
    assert at[[0, 1, 2, 3, 4], 1].all() and not at[:, 0].any() and not at[[5, 6]].any()


def test_endpoint_rf_tie_taints_the_seed():
    g = graph(3, [(0, 1, 2.0), (1, 2, 3.0)], ep=[2], rat=[6.0], src_mean=np.zeros((3, 2)))   # R and F slack 1
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    assert not ft.any() and at.all()


def test_endpoint_slack_at_zero_taints_the_seed():
    # no merge tie; z's slack is exactly 0 (the TNS seed is a kink): the adjoint of z is
    # uncertain, so its unambiguous upstream chain is flagged winner by winner
    arcs = [(0, 1, 2.0), (1, 2, 3.0)]
    g = graph(3, arcs, ep=[2], rat=[5.5])                # A = (5, 5.5): fall slack exactly 0
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    assert not ft.any()
    assert at.all()
    g2 = graph(3, arcs, ep=[2], rat=[6.5])               # slack 1: certain seed, nothing flagged
    ft2, at2 = oracle.tie_taint(g2, NS, eps=1e-3, margin=0.05)
    assert not ft2.any() and not at2.any()
