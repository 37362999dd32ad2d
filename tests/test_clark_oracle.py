"""Pins for the Clark moment-matching oracle -- no GPU.

orc_clark_forward folds Clark's max of two independent Gaussians over a pin's
candidates in canonical order (reading R20); orc_clark_backward differentiates
that fold.  Checked against:
* the closed form for two iid inputs: E = mu + sigma/sqrt(pi), Var = sigma^2 (1 - 1/pi);
* the EXACT first two moments of max(X, Y) for independent Gaussians by
  numerical integration (scipy.integrate.quad) -- Clark's formulas are exact
  for two inputs -- and, iterated in the canonical candidate order, for 3-4
  inputs (pins the fold order and the unateness routing);
* single-fanin chains (moments add, Eq 1-2) and the sigma -> 0 limit (hard max);
* central finite differences of a smooth endpoint loss for every gradient
  output (arc mean, arc sigma, source mean, source sigma).
"""
import types

import numpy as np
import pytest
from scipy import integrate, stats

import oracle
from tests import bruteforce as bf

NS = 3.0


def exact_max_moments(m1, s1, m2, s2):
    """E[max(X, Y)], Var[max(X, Y)] for independent X ~ N(m1, s1^2), Y ~ N(m2, s2^2), by quadrature."""
    if s1 == 0 and s2 == 0:
        return max(m1, m2), 0.0
    # density of Z = max(X, Y): f_X F_Y + f_Y F_X
    def pdf(z):
        fx = stats.norm.pdf(z, m1, s1) if s1 > 0 else 0.0
        fy = stats.norm.pdf(z, m2, s2) if s2 > 0 else 0.0
        Fx = stats.norm.cdf(z, m1, s1) if s1 > 0 else float(z >= m1)
        Fy = stats.norm.cdf(z, m2, s2) if s2 > 0 else float(z >= m2)
        return fx * Fy + fy * Fx
    lo = min(m1 - 12 * s1, m2 - 12 * s2)
    hi = max(m1 + 12 * s1, m2 + 12 * s2)
    pts = [m1, m2]
    e1 = integrate.quad(lambda z: z * pdf(z), lo, hi, points=pts, epsabs=1e-13, epsrel=1e-13, limit=400)[0]
    e2 = integrate.quad(lambda z: (z - e1) ** 2 * pdf(z), lo, hi, points=pts, epsabs=1e-13, epsrel=1e-13,
                        limit=400)[0]
    return e1, e2


def star_graph(src, arcs):
    """Sources 0..n-1 with (mu, sigma) per rf, a sink n fed by arcs (src, unate, mean[2], sigma[2]) in arc-id order."""
    n = len(src)
    E = len(arcs)
    return types.SimpleNamespace(
        num_pins=n + 1, arc_from=np.array([a[0] for a in arcs], np.int32), arc_to=np.full(E, n, np.int32),
        arc_unate=np.array([a[1] for a in arcs], np.uint8),
        arc_mean=np.array([a[2] for a in arcs], float).reshape(E, 2),
        arc_sigma=np.array([a[3] for a in arcs], float).reshape(E, 2),
        src_mean=np.array([s[0] for s in src] + [(0.0, 0.0)], float),
        src_sigma=np.array([s[1] for s in src] + [(0.0, 0.0)], float),
        ep_pin=np.array([n], np.int32), ep_rat=np.array([[100.0, 100.0]]))


def test_clark_iid_closed_form():
    mu, sg = 10.0, 2.0
    g = star_graph([((mu, mu), (sg, sg)), ((mu, mu), (sg, sg))],
                   [(0, 0, (0, 0), (0, 0)), (1, 0, (0, 0), (0, 0))])
    f = oracle.clark_forward(g, NS)
    assert f["mu"][2, 0] == pytest.approx(mu + sg / np.sqrt(np.pi), abs=1e-12)
    assert f["sigma"][2, 0] ** 2 == pytest.approx(sg * sg * (1 - 1 / np.pi), abs=1e-12)


@pytest.mark.parametrize("seed", range(8))
def test_clark_two_inputs_exact_moments(seed):
    rng = np.random.default_rng(seed)
    m = rng.uniform(0, 20, 2)
    s = rng.uniform(0.2, 4, 2)
    d = rng.uniform(0, 10, 2)
    ds = rng.uniform(0, 2, 2)
    g = star_graph([((m[0], 0), (s[0], 0)), ((m[1], 0), (s[1], 0))],
                   [(0, 0, (d[0], 0), (ds[0], 0)), (1, 0, (d[1], 0), (ds[1], 0))])
    f = oracle.clark_forward(g, NS)
    e1, var = exact_max_moments(m[0] + d[0], np.hypot(s[0], ds[0]), m[1] + d[1], np.hypot(s[1], ds[1]))
    assert f["mu"][2, 0] == pytest.approx(e1, rel=1e-9, abs=1e-9)
    assert f["sigma"][2, 0] ** 2 == pytest.approx(var, rel=1e-7, abs=1e-9)


@pytest.mark.parametrize("seed", range(6))
def test_clark_fold_order_and_unateness(seed):
    """3-4 inputs with mixed unateness: the oracle equals the exact two-input max moments iterated in the
    canonical order (arc id ascending, s = rf before ~rf) with the Gaussian re-approximation after each step."""
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(3, 5))
    src = [((rng.uniform(0, 20), rng.uniform(0, 20)), (rng.uniform(0.5, 3), rng.uniform(0.5, 3))) for _ in range(n)]
    arcs = []
    for k in range(n):
        arcs.append((k, int(rng.integers(0, 3)), (rng.uniform(0, 5), rng.uniform(0, 5)),
                     (rng.uniform(0, 1), rng.uniform(0, 1))))
    g = star_graph(src, arcs)
    f = oracle.clark_forward(g, NS)
    for rf in (0, 1):
        cands = []
        for e, (j, u, am, asg) in enumerate(arcs):
            for s in bf.source_transitions(rf, u):
                cands.append((src[j][0][s] + am[rf], np.hypot(src[j][1][s], asg[rf])))
        mu, sd = cands[0]
        for m2, s2 in cands[1:]:
            mu, var = exact_max_moments(mu, sd, m2, s2)
            sd = np.sqrt(var)
        assert f["mu"][n, rf] == pytest.approx(mu, rel=1e-8, abs=1e-8)
        assert f["sigma"][n, rf] == pytest.approx(sd, rel=1e-6, abs=1e-8)


def test_clark_chain_adds_moments():
    g = types.SimpleNamespace(
        num_pins=3, arc_from=np.array([0, 1], np.int32), arc_to=np.array([1, 2], np.int32),
        arc_unate=np.array([0, 1], np.uint8), arc_mean=np.array([[3.0, 4.0], [5.0, 6.0]]),
        arc_sigma=np.array([[0.3, 0.4], [1.2, 0.5]]), src_mean=np.array([[1.0, 2.0], [0, 0], [0, 0]]),
        src_sigma=np.array([[0.1, 0.2], [0, 0], [0, 0]]), ep_pin=np.array([2], np.int32),
        ep_rat=np.array([[50.0, 50.0]]))
    f = oracle.clark_forward(g, NS)
    # pin 2 rise <- arc 1 (NEG) from pin 1 fall <- arc 0 (POS) from pin 0 fall
    assert f["mu"][2, 0] == pytest.approx(2.0 + 4.0 + 5.0, abs=1e-12)
    assert f["sigma"][2, 0] == pytest.approx(np.sqrt(0.2 ** 2 + 0.4 ** 2 + 1.2 ** 2), abs=1e-12)
    assert f["A"][2, 0] == pytest.approx(f["mu"][2, 0] + NS * f["sigma"][2, 0], abs=1e-12)


@pytest.mark.parametrize("seed", range(6))
def test_clark_sigma0_is_hard_max(seed):
    g = bf.tiny_dag(seed, n_pins=9, p_edge=0.4, sigma0=True)
    f = oracle.clark_forward(g, NS)
    h = oracle.forward(g, NS, 0.0)
    assert np.array_equal(f["A"], h["A"])
    assert (f["sigma"] == 0).all()


def _loss(g, w):
    f = oracle.clark_forward(g, NS)
    s = np.minimum(g.ep_rat[:, 0] - f["A"][g.ep_pin, 0], g.ep_rat[:, 1] - f["A"][g.ep_pin, 1])
    return float(np.dot(w, s))


@pytest.mark.parametrize("seed", range(8))
def test_clark_gradients_central_fd(seed):
    """Every gradient output against central differences of L = sum_k w_k slack_k (smooth away from rf ties)."""
    g = bf.tiny_dag(seed, n_pins=8, p_edge=0.45, n_ep=3)
    g.src_sigma = np.maximum(g.src_sigma, 0.5)           # V > 0 everywhere: Clark is smooth
    g.arc_sigma = np.maximum(g.arc_sigma, 0.2)
    w = np.random.default_rng(seed).uniform(0.5, 2.0, len(g.ep_pin))
    b = oracle.clark_backward(g, NS, dslack=w)
    h = 1e-6
    for name, arr, grad in [("arc_mean", "arc_mean", "d_mean"), ("arc_sigma", "arc_sigma", "d_sigma"),
                            ("src_mean", "src_mean", "d_src_mean"), ("src_sigma", "src_sigma", "d_src_sigma")]:
        base = getattr(g, arr).copy()
        for idx in np.ndindex(*base.shape):
            if arr.startswith("src"):
                indeg = np.bincount(g.arc_to, minlength=g.num_pins)
                if indeg[idx[0]] > 0:
                    continue
            gp = base.copy(); gp[idx] += h
            gm = base.copy(); gm[idx] -= h
            setattr(g, arr, gp); lp = _loss(g, w)
            setattr(g, arr, gm); lm = _loss(g, w)
            setattr(g, arr, base)
            fd = (lp - lm) / (2 * h)
            assert b[grad][idx] == pytest.approx(fd, rel=2e-5, abs=2e-6), (name, idx)
