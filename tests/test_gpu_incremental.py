"""Incremental re-propagation: after
insta_update_arcs(incremental=1), insta_forward recomputes only the changed
cone and must equal a full forward on the updated graph bit for bit."""
import types

import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth

pytestmark = pytest.mark.gpu


def fresh(g, mean, sigma, tau, schedule=0):
    h = types.SimpleNamespace(**vars(g))
    h.arc_mean, h.arc_sigma = mean, sigma
    H = insta.Graph(h)
    s = H.forward(3.0, tau, schedule)
    A, m, sg = (x.cpu().numpy() for x in H.arrivals())
    d = H.backward().cpu().numpy()
    sl = H.slack()[0].cpu().numpy()
    H.close()
    return s, A, m, sg, d, sl


CONE = 10 ** 9   # cone_max: take the cone pass whatever the update size


@pytest.mark.parametrize("tau", [0.0, 1.0])
@pytest.mark.parametrize("schedule", [0, 2, 3])
def test_incremental_equals_full(tau, schedule):
    g = synth.generate("C2")
    mean, sigma = g.arc_mean.copy(), g.arc_sigma.copy()
    G = insta.Graph(g)
    G.forward(3.0, tau, schedule)
    for step in range(3):
        ids, m, s = synth.sizing_step(g, step, frac=0.002)
        mean[ids], sigma[ids] = m, s
        G.update_arcs(ids, m, s, incremental=True)
        summ = G.forward(3.0, tau, schedule, cone_max=CONE)
        n_re = G.last_forward_stats()
        assert 0 < n_re < g.num_pins
        A, mm, sg = (x.cpu().numpy() for x in G.arrivals())
        d = G.backward().cpu().numpy()
        sl = G.slack()[0].cpu().numpy()
        s2, A2, m2, sg2, d2, sl2 = fresh(g, mean, sigma, tau, schedule)
        assert np.array_equal(A, A2) and np.array_equal(mm, m2) and np.array_equal(sg, sg2)
        assert np.array_equal(sl, sl2)
        assert summ.tns == s2.tns and summ.wns == s2.wns and summ.num_violations == s2.num_violations
        assert np.array_equal(d, d2)
    G.close()


def test_incremental_against_oracle_and_cone_size():
    g = synth.generate("C2")
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    ids, m, s = synth.sizing_step(g, 0, frac=0.001)
    G.update_arcs(ids, m, s, incremental=True)
    summ = G.forward(3.0, 0.0, cone_max=CONE)
    n_re = G.last_forward_stats()
    h = types.SimpleNamespace(**vars(g))
    h.arc_mean, h.arc_sigma = g.arc_mean.copy(), g.arc_sigma.copy()
    h.arc_mean[ids], h.arc_sigma[ids] = m, s
    o = oracle.slack(h, oracle.forward(h, 3.0, 0.0)["A"])
    assert summ.tns == pytest.approx(o["tns"], rel=1e-6)
    # the cone of a 0.1% update is a strict subset of the graph
    assert n_re < 0.9 * g.num_pins
    G.close()


def test_incremental_fallbacks_to_full():
    g = synth.generate("C1")
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    ids = np.array([0, 5, 9], np.int32)
    # no-op update: sinks recomputed, nothing changes, result identical
    A0 = G.arrivals()[0].cpu().numpy()
    G.update_arcs(ids, g.arc_mean[ids], g.arc_sigma[ids], incremental=True)
    G.forward(3.0, 0.0)
    assert G.last_forward_stats() <= 3 * 5   # the 3 heads evaluating the arcs (+ their folded input pins)
    assert np.array_equal(G.arrivals()[0].cpu().numpy(), A0)
    # option change -> full pass
    G.update_arcs(ids, g.arc_mean[ids] * 1.1, g.arc_sigma[ids], incremental=True)
    G.forward(3.0, 1.0)
    assert G.last_forward_stats() == g.num_pins
    # a non-incremental update forces a full pass
    G.update_arcs(ids, g.arc_mean[ids], g.arc_sigma[ids], incremental=False)
    G.forward(3.0, 1.0)
    assert G.last_forward_stats() == g.num_pins
    G.close()


def test_default_policy_full_pass_for_large_batches():
    """Above cone_max re-annotated arcs (default max(64, E/1e5)) the forward is a full pass
    (include/insta.h), below it the cone pass; both equal a fresh graph bit for bit."""
    g = synth.generate("C2")
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    ids, m, s = synth.sizing_step(g, 5, frac=0.01)
    assert len(ids) > 64
    G.update_arcs(ids, m, s, incremental=True)
    G.forward(3.0, 0.0)
    assert G.last_forward_stats() == g.num_pins          # full pass
    ids2 = ids[:4]
    G.update_arcs(ids2, m[:4] * np.float32(1.01), s[:4], incremental=True)
    G.forward(3.0, 0.0)
    assert G.last_forward_stats() < g.num_pins           # cone pass
    A = G.arrivals()[0].cpu().numpy()
    mean, sigma = g.arc_mean.copy(), g.arc_sigma.copy()
    mean[ids], sigma[ids] = m, s
    mean[ids2] = m[:4] * np.float32(1.01)
    s2, A2, _, _, _, _ = fresh(g, mean, sigma, 0.0)
    assert np.array_equal(A, A2)
    G.close()


@pytest.mark.slow
def test_c3_incremental_steps():
    """C3 (BASELINE configs[2]): 1 % sizing steps, cone pass (forced) and default policy: bit-identical
    to a fresh full pass on the updated arcs, TNS equal to the fp64 oracle's."""
    g = synth.generate("C3")
    mean, sigma = g.arc_mean.copy(), g.arc_sigma.copy()
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    for step in range(3):
        ids, m, s = synth.sizing_step(g, step, frac=0.01)
        mean[ids], sigma[ids] = m, s
        G.update_arcs(ids, m, s, incremental=True)
        summ = G.forward(3.0, 0.0, cone_max=CONE if step % 2 == 0 else 0)
        A = G.arrivals()[0].cpu().numpy()
        sl = G.slack()[0].cpu().numpy()
    d = G.backward().cpu().numpy()
    s2, A2, _, _, d2, sl2 = fresh(g, mean, sigma, 0.0)
    assert np.array_equal(A, A2) and np.array_equal(sl, sl2) and np.array_equal(d, d2)
    assert summ.tns == s2.tns
    h = types.SimpleNamespace(**vars(g))
    h.arc_mean, h.arc_sigma = mean, sigma
    o = oracle.slack(h, oracle.forward(h, 3.0, 0.0)["A"])
    assert summ.tns == pytest.approx(o["tns"], rel=1e-6)
    G.close()
