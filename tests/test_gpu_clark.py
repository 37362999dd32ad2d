"""GPU parity of the Clark moment-matching path vs the fp64 oracle.

Both sides are fp64 with the same closed forms, so the tolerances are the north
star's (arrival / slack: max(1e-4 |x|, 1e-3 ps); gradients: 1e-3 max(|g|, 1))
and hold with orders of magnitude to spare; sigma = 0 reduces to the hard max.
"""
import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth
from tests import bruteforce as bf

pytestmark = pytest.mark.gpu
NS = 3.0


def within(x, ref, rel=1e-4, ab=1e-3):
    x = np.asarray(x, np.float64)
    return np.abs(x - ref) <= np.maximum(rel * np.abs(ref), ab)


def run(g, seed=None):
    G = insta.Graph(g)
    s = G.clark_forward(NS)
    r = {k: v.cpu().numpy() for k, v in G.clark_results().items()}
    dm, ds, dsrc = (x.cpu().numpy() for x in G.clark_backward(ep_seed=seed, want_sigma=True, want_src=True))
    G.close()
    return s, r, dm, ds, dsrc


@pytest.mark.parametrize("seed", range(8))
def test_clark_tiny(seed):
    g = bf.tiny_dag(seed, n_pins=9, p_edge=0.45, n_ep=4)
    s, r, dm, ds, dsrc = run(g)
    f = oracle.clark_forward(g, NS)
    b = oracle.clark_backward(g, NS)
    assert within(r["A"], f["A"]).all()
    assert within(r["mean"], f["mu"]).all()
    assert within(r["sigma"], f["sigma"]).all()
    assert within(dm, b["d_mean"], 1e-3, 1e-3).all()
    assert within(ds, b["d_sigma"], 1e-3, 1e-3).all()
    assert within(dsrc, b["d_src_mean"], 1e-3, 1e-3).all()


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_clark_configs(cfg):
    g = synth.generate(cfg)
    s, r, dm, ds, dsrc = run(g)
    f = oracle.clark_forward(g, NS)
    b = oracle.clark_backward(g, NS)
    A = r["A"]
    assert within(A, f["A"]).all(), np.abs(A - f["A"]).max()
    sl = np.minimum(g.ep_rat[:, 0] - f["A"][g.ep_pin, 0], g.ep_rat[:, 1] - f["A"][g.ep_pin, 1])
    assert within(r["slack"], sl).all()
    tns = float(np.minimum(sl, 0).sum())
    assert abs(s.tns - tns) <= 1e-6 * abs(tns) + 1e-3
    assert s.num_violations == int((sl < 0).sum())
    assert within(dm, b["d_mean"], 1e-3, 1e-3).all(), np.abs(dm - b["d_mean"]).max()
    assert within(ds, b["d_sigma"], 1e-3, 1e-3).all(), np.abs(ds - b["d_sigma"]).max()


def test_clark_custom_seed_and_sigma0():
    g = synth.generate("C1")
    w = np.random.default_rng(3).uniform(0, 2, g.num_endpoints).astype(np.float32)
    _, _, dm, _, _ = run(g, seed=w)
    b = oracle.clark_backward(g, NS, dslack=w.astype(np.float64))
    assert within(dm, b["d_mean"], 1e-3, 1e-3).all()
    # sigma = 0 everywhere: the hard max (dyadic values: exact)
    h = synth.generate("C1", dyadic=True)
    G = insta.Graph(h)
    G.clark_forward(NS)
    A = G.clark_results()["A"].cpu().numpy()
    G.forward(NS, 0.0)
    A0 = G.arrivals()[0].cpu().numpy()
    G.close()
    assert np.array_equal(A, A0)


def test_clark_errors():
    g = synth.generate("C1")
    G = insta.Graph(g)
    with pytest.raises(insta.InstaError, match="E_STATE"):
        G.clark_results()
    with pytest.raises(insta.InstaError, match="E_STATE"):
        G.clark_backward()
    G.clark_forward(NS)
    G.update_arcs(np.array([0]), g.arc_mean[:1], g.arc_sigma[:1])
    with pytest.raises(insta.InstaError, match="E_STATE"):
        G.clark_backward()
    G.close()
