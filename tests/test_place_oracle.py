"""Pins for the Eq 7 timing-objective oracle -- no GPU.

Against things other than the formula itself: a hand example, central finite
differences of L for every pin coordinate (generic positions, no ties),
translation invariance (L depends on differences only: the gradient sums to
zero), positive homogeneity L(a x, a y) = a L, and linearity in the weights.
"""
import types

import numpy as np
import pytest

import oracle
from paper_conf_dac_lugklr25_b200 import synth


def _graph(n, af, at):
    E = len(af)
    return types.SimpleNamespace(num_pins=n, arc_from=np.asarray(af, np.int32), arc_to=np.asarray(at, np.int32),
                                 arc_unate=np.zeros(E, np.uint8), arc_mean=np.ones((E, 2)), arc_sigma=np.zeros((E, 2)),
                                 src_mean=None, src_sigma=None, ep_pin=np.zeros(0, np.int32), ep_rat=np.zeros((0, 2)))


def test_hand_example():
    # arcs 0->1 (w 2) and 1->2 (w 0.5); pins at (0,0), (3,-1), (1,4); lambda 0.1
    g = _graph(3, [0, 1], [1, 2])
    L, gx, gy = oracle.timing_loss(g, [0, 3, 1], [0, -1, 4], [2.0, 0.5], 0.1)
    assert L == pytest.approx(0.1 * (2 * (3 + 1) + 0.5 * (2 + 5)))
    assert gx == pytest.approx([0.1 * 2 * -1, 0.1 * (2 * 1 + 0.5 * 1), 0.1 * 0.5 * -1])
    assert gy == pytest.approx([0.1 * 2 * 1, 0.1 * (2 * -1 + 0.5 * -1), 0.1 * 0.5 * 1])


@pytest.mark.parametrize("seed", range(4))
def test_fd_and_invariances(seed):
    g = synth.generate("C1")
    rng = np.random.default_rng(seed)
    N, E = g.num_pins, g.num_arcs
    x, y = rng.uniform(0, 100, N), rng.uniform(0, 100, N)
    w = np.where(rng.random(E) < 0.3, rng.uniform(0, 2, E), 0.0)
    lam = 1e-3
    L, gx, gy = oracle.timing_loss(g, x, y, w, lam)
    h = 1e-4   # L is piecewise linear: exact away from kinks (|x_f - x_t| > h)
    for p in rng.choice(N, 40, replace=False):
        for arr, grad in ((x, gx), (y, gy)):
            arr[p] += h; lp = oracle.timing_loss(g, x, y, w, lam)[0]
            arr[p] -= 2 * h; lm = oracle.timing_loss(g, x, y, w, lam)[0]
            arr[p] += h
            assert grad[p] == pytest.approx((lp - lm) / (2 * h), rel=1e-6, abs=1e-8)
    assert abs(gx.sum()) < 1e-9 and abs(gy.sum()) < 1e-9
    assert oracle.timing_loss(g, x + 7.5, y - 3.0, w, lam)[0] == pytest.approx(L, rel=1e-12)
    assert oracle.timing_loss(g, 2.5 * x, 2.5 * y, w, lam)[0] == pytest.approx(2.5 * L, rel=1e-12)
    w2 = rng.uniform(0, 1, E)
    assert oracle.timing_loss(g, x, y, w + w2, lam)[0] == pytest.approx(L + oracle.timing_loss(g, x, y, w2, lam)[0],
                                                                       rel=1e-12)
