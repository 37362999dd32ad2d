"""INSTA-Size device steps and loop on the GPU.

* insta_stage_gradients vs the oracle's stage composition (R22) of the same
  gradient; insta_select_stages vs a stable numpy selection + sort;
* the sizing loop: every committed trial strictly improves TNS, TNS improves
  overall, rollbacks restore the previous TNS exactly (the incremental pass is
  bit-identical to a full one), and the final state's TNS equals the fp64
  oracle's on the final annotation.
"""
import types

import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import size, synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("cfg,tau", [("C1", 0.0), ("C2", 0.0), ("C2", 1.0)])
def test_stage_gradients_and_selection(cfg, tau):
    g = synth.generate(cfg)
    G = insta.Graph(g)
    G.forward(3.0, tau)
    d = G.backward()
    sg = G.stage_gradients(d)
    thr = 0.05
    sel = G.select_stages(sg, thr).cpu().numpy()
    sg_h, d_h = sg.cpu().numpy(), d.cpu().numpy().astype(np.float64)
    G.close()
    ref = oracle.stage_gradients(g, d_h)
    assert np.allclose(sg_h, ref, rtol=1e-6, atol=1e-6)
    cand = np.nonzero(sg_h < -thr)[0]
    expect = cand[np.argsort(sg_h[cand], kind="stable")]
    assert np.array_equal(sel, expect)
    assert (g.arc_class[sel] == synth.CELL).all()


def test_insta_size_loop_c2():
    g = synth.generate("C2")
    G = insta.Graph(g)
    r = size.insta_size(G, g, iterations=2, per_iter=15, max_trials=60)
    G.close()
    assert r.commits > 0 and r.tns > r.tns0
    best = r.tns0
    for it, trial, tns, ok in r.history:
        if ok:
            assert tns > best
            best = tns
        else:
            assert tns <= best
    # the end state against the fp64 oracle on the final annotation
    h = types.SimpleNamespace(**vars(g))
    h.arc_mean, h.arc_sigma = r.arc_mean, r.arc_sigma
    f = oracle.forward(h, 3.0, 0.0)
    o = oracle.slack(h, f["A"])
    assert abs(r.tns - o["tns"]) <= 1e-6 * abs(o["tns"]) + 1e-3, (r.tns, o["tns"])
