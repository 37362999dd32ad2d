"""Pin for the INSTA-Size stage gradient (reading R22) -- no GPU.

A stage gradient is the directional derivative of TNS when a cell arc and its
driving net arc are delayed together (both transitions): checked against
central finite differences of the oracle's forward TNS (LSE tau = 1 ps, smooth),
and net arcs / stage structure against the graph.
"""
import numpy as np
import pytest

import oracle
from paper_conf_dac_lugklr25_b200 import synth

NS, TAU = 3.0, 1.0


def _tns(g):
    f = oracle.forward(g, NS, TAU)
    return oracle.slack(g, f["A"])["tns"]


def test_stage_gradient_is_directional_derivative():
    g = synth.generate("C1")
    b = oracle.backward(g, NS, TAU)
    sg = oracle.stage_gradients(g, b["d_mean"])
    assert (sg[g.arc_class == synth.NET] == 0).all()
    cell = np.nonzero((g.arc_class == synth.CELL) & (np.abs(sg) > 1e-3))[0]
    assert cell.size > 10
    indeg = np.bincount(g.arc_to, minlength=g.num_pins)
    rng = np.random.default_rng(0)
    base = g.arc_mean.astype(np.float64).copy()
    g.arc_mean = base
    h = 1e-4
    for e in rng.choice(cell, 12, replace=False):
        p = g.arc_from[e]
        arcs = [e]
        if indeg[p] == 1:
            n = int(np.nonzero(g.arc_to == p)[0][0])
            if g.arc_class[n] == synth.NET:
                arcs.append(n)
        d = np.zeros_like(base)
        d[arcs] = 1.0
        g.arc_mean = base + h * d
        tp = _tns(g)
        g.arc_mean = base - h * d
        tm = _tns(g)
        g.arc_mean = base
        assert sg[e] == pytest.approx((tp - tm) / (2 * h), rel=1e-4, abs=1e-6)
