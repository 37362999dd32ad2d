"""Batched scenario evaluation (insta_forward_batch).

Each scenario is checked against the single-scenario path run on the
scenario's materialized graph (fp32 derates, overrides) -- arrivals are the
same arithmetic, so WNS and violation counts must match exactly and TNS to
summation-order rounding -- and against the fp64 oracle.
"""
import types

import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth

pytestmark = pytest.mark.gpu


def scenarios(g, n, seed=7):
    rng = np.random.default_rng(seed)
    cell = np.nonzero(g.arc_class == synth.CELL)[0]
    sinks = g.arc_to[cell]
    out = []
    for s in range(n):
        if s % 2 == 0:
            ns, dc, dn = synth.ocv_scenario(s)
            out.append(dict(n_sigma=ns, derate_cell=dc, derate_net=dn))
        else:   # sizing candidate: one cell's arcs scaled
            pin = sinks[rng.integers(sinks.size)]
            ids = cell[sinks == pin].astype(np.int32)
            f = np.float32(rng.uniform(0.75, 1.05))
            out.append(dict(n_sigma=3.0, derate_cell=1.0, derate_net=1.0, delta_arc=ids,
                            delta_mean=(g.arc_mean[ids] * f).astype(np.float32),
                            delta_sigma=(g.arc_sigma[ids] * f).astype(np.float32)))
    return out


def materialize(g, sc):
    d = np.where(g.arc_class == synth.CELL, np.float32(sc["derate_cell"]), np.float32(sc["derate_net"]))
    d = d.astype(np.float32)[:, None]
    m = (g.arc_mean * d).astype(np.float32)
    s = (g.arc_sigma * d).astype(np.float32)
    if sc.get("delta_arc") is not None:
        m[sc["delta_arc"]] = sc["delta_mean"]
        s[sc["delta_arc"]] = sc["delta_sigma"]
    h = types.SimpleNamespace(**vars(g))
    h.arc_mean, h.arc_sigma = m, s
    return h


@pytest.mark.parametrize("cfg,tau,nsc", [("C2", 0.0, 40), ("C1", 1.0, 37), ("C1", 0.0, 5)])
def test_batch_matches_single_scenario_runs(cfg, tau, nsc):
    g = synth.generate(cfg)
    scs = scenarios(g, nsc)
    G = insta.Graph(g)
    G.forward(3.0, tau)
    A_before = G.arrivals()[0].cpu().numpy()
    summ, dsum = G.forward_batch(scs, tau=tau, want_grad=True)
    summ = summ.cpu().numpy()
    dsum = dsum.cpu().numpy()
    assert np.array_equal(G.arrivals()[0].cpu().numpy(), A_before)   # single-scenario state untouched
    G.close()
    gsum = np.zeros((g.num_arcs, 2), np.float64)
    for k, sc in enumerate(scs):
        h = materialize(g, sc)
        H = insta.Graph(h)
        s = H.forward(sc["n_sigma"], tau)
        d = H.backward().cpu().numpy()
        H.close()
        assert summ[k, 0] == s.wns, k
        assert summ[k, 2] == s.num_violations, k
        assert summ[k, 1] == pytest.approx(s.tns, rel=1e-12, abs=1e-9), k
        gsum += d
    if tau == 0.0:
        assert np.array_equal(dsum, gsum.astype(np.float32))   # integer path counts: exact
    else:
        assert np.allclose(dsum, gsum, rtol=1e-5, atol=1e-5)


def test_batch_against_oracle():
    g = synth.generate("C1")
    scs = scenarios(g, 6, seed=3)
    G = insta.Graph(g)
    summ, dsum = G.forward_batch(scs, tau=1.0, want_grad=True)
    summ = summ.cpu().numpy()
    dsum = dsum.cpu().numpy()
    G.close()
    want = np.zeros((g.num_arcs, 2))
    for k, sc in enumerate(scs):
        h = materialize(g, sc)
        f = oracle.forward(h, sc["n_sigma"], 1.0)
        o = oracle.slack(h, f["A"])
        assert summ[k, 1] == pytest.approx(o["tns"], rel=1e-5, abs=1e-3)
        assert summ[k, 2] == o["num_viol"]
        want += oracle.backward(h, sc["n_sigma"], 1.0)["d_mean"]
    assert np.abs(dsum - want).max() <= 1e-3 * max(1.0, np.abs(want).max())


def test_batch_forward_only_and_errors():
    g = synth.generate("C1")
    G = insta.Graph(g)
    summ, dsum = G.forward_batch([dict(n_sigma=3.0, derate_cell=1.0, derate_net=1.0)], tau=0.0)
    assert dsum is None
    s = G.forward(3.0, 0.0)
    assert summ.cpu().numpy()[0, 1] == pytest.approx(s.tns, rel=1e-12)
    with pytest.raises(insta.InstaError, match="E_ARG"):
        G.forward_batch([dict(n_sigma=-1.0)])
    with pytest.raises(insta.InstaError, match="E_ARG"):
        G.forward_batch([dict(delta_arc=np.array([10 ** 8]), delta_mean=np.zeros((1, 2)), delta_sigma=np.zeros((1, 2)))])
    G.close()


@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_batch_sizing_candidates_with_input_nets(tau):
    """C5 sizing candidates (synth.sizing_scenario): a cell's arcs AND its input net arcs are
    overridden in one scenario, so a cell arc and the net arc behind its folded input pin share an
    entry (override bits 1 and 3 of one flag byte, set concurrently).  Every scenario equals
    insta_forward on its materialized graph, and clearing the overrides restores the base."""
    g = synth.generate("C2")
    scs = [synth.sizing_scenario(g, s) for s in range(512, 512 + 64)]
    assert any(len(sc["delta_arc"]) > 4 for sc in scs)
    G = insta.Graph(g)
    base = G.forward(3.0, tau)
    summ, _ = G.forward_batch(scs, tau=tau)
    summ = summ.cpu().numpy()
    again, _ = G.forward_batch([dict(n_sigma=3.0, derate_cell=1.0, derate_net=1.0)], tau=tau)
    assert again.cpu().numpy()[0, 1] == pytest.approx(base.tns, rel=1e-12)   # no stale override bits
    G.close()
    for k, sc in enumerate(scs):
        H = insta.Graph(materialize(g, sc))
        s = H.forward(3.0, tau)
        H.close()
        assert summ[k, 0] == s.wns and summ[k, 2] == s.num_violations, k
        assert summ[k, 1] == pytest.approx(s.tns, rel=1e-12, abs=1e-9), k


@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_eval_candidates_cone(tau):
    """insta_eval_candidates (C5 sizing candidates through the cone pass): every candidate's summary equals
    insta_forward on its materialized graph bit for bit, and the graph returns to its base state."""
    g = synth.generate("C2")
    scs = [synth.sizing_scenario(g, s) for s in range(512, 512 + 24)]
    # an empty candidate (the base state) and one listing an arc twice with the same record
    scs.insert(3, dict(n_sigma=3.0, derate_cell=1.0, derate_net=1.0, delta_arc=np.zeros(0, np.int32),
                       delta_mean=np.zeros((0, 2), np.float32), delta_sigma=np.zeros((0, 2), np.float32)))
    d = scs[5]
    scs.insert(6, dict(d, delta_arc=np.concatenate([d["delta_arc"], d["delta_arc"][:1]]),
                       delta_mean=np.concatenate([d["delta_mean"], d["delta_mean"][:1]]),
                       delta_sigma=np.concatenate([d["delta_sigma"], d["delta_sigma"][:1]])))
    G = insta.Graph(g)
    base = G.forward(3.0, tau)
    A0 = G.arrivals()[0].cpu().numpy()
    sl0 = G.slack()[0].cpu().numpy()
    d0 = G.backward().cpu().numpy()
    summ = G.eval_candidates(scs).cpu().numpy()
    assert np.array_equal(G.arrivals()[0].cpu().numpy(), A0)
    assert np.array_equal(G.slack()[0].cpu().numpy(), sl0)
    assert np.array_equal(G.backward().cpu().numpy(), d0)
    assert G.summary().tns == base.tns
    assert summ[3, 1] == base.tns and summ[3, 0] == base.wns
    # a second batch on the restored state gives the same summaries
    assert np.array_equal(G.eval_candidates(scs[:8]).cpu().numpy(), summ[:8])
    G.close()
    for k, sc in enumerate(scs):
        H = insta.Graph(materialize(g, sc))
        s = H.forward(3.0, tau)
        H.close()
        assert summ[k, 0] == s.wns and summ[k, 1] == s.tns and summ[k, 2] == s.num_violations, k


@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_batch_and_candidates_against_oracle_c2(tau):
    """C2 (200k pins): OCV scenarios (insta_forward_batch) and one-cell sizing candidates
    (insta_eval_candidates) against the fp64 oracle on each materialized graph -- TNS / WNS within
    the slack tolerance, violation counts equal."""
    g = synth.generate("C2")
    ocv = scenarios(g, 6, seed=11)
    cand = [synth.sizing_scenario(g, s) for s in range(700, 706)]
    G = insta.Graph(g)
    s_ocv = G.forward_batch(ocv, tau=tau, want_grad=False)[0].cpu().numpy()
    G.forward(3.0, tau)
    s_cand = G.eval_candidates(cand).cpu().numpy()
    G.close()
    for summ, scs in ((s_ocv, ocv), (s_cand, cand)):
        for k, sc in enumerate(scs):
            h = materialize(g, sc)
            f = oracle.forward(h, sc["n_sigma"], tau)
            o = oracle.slack(h, f["A"])
            assert summ[k, 1] == pytest.approx(o["tns"], rel=1e-5, abs=1e-3), (k, summ[k], o["tns"])
            assert summ[k, 0] == pytest.approx(o["wns"], rel=1e-4, abs=1e-3)
            assert abs(summ[k, 2] - o["num_viol"]) <= 1   # a slack within rounding of 0 may flip
