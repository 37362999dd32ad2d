"""GPU parity: the CUDA path (through the C ABI) vs the fp64 CPU oracle.

Tolerances (BASELINE.json north_star):
  levelization / CSR: bit-exact;
  arrival, slack: |x - x_ref| <= max(1e-4 |x_ref|, 1e-3 ps);
  gradients: |g - g_ref| <= 1e-3 max(|g_ref|, 1) for tau = 0 (tie-free arcs) and tau >= 1 ps;
             ||g - g_ref|| <= 1e-3 ||g_ref|| ... reported for tau = 0.01 (see test);
  dyadic mode (mu on a 2^-6 grid, sigma = 0): bit-exact, ties included.
Near-tie arcs in hard mode are excluded using the oracle's taint mask
(oracle.tie_taint) and must stay a small fraction.
"""
import types

import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth
from tests import bruteforce as bf

pytestmark = pytest.mark.gpu
NS = 3.0


def tol_ok(x, ref, mask=None):
    err = np.abs(np.asarray(x, np.float64) - ref)
    lim = np.maximum(1e-4 * np.abs(ref), 1e-3)
    bad = err > lim
    if mask is not None:
        bad &= ~mask
    return bad


def run_gpu(g, tau=0.0, schedule=0, seed=None, want_src=False):
    G = insta.Graph(g)
    s = G.forward(NS, tau, schedule)
    A, mu, sig = (x.cpu().numpy() for x in G.arrivals())
    sl, rf = (x.cpu().numpy() for x in G.slack())
    out = G.backward(ep_seed=seed, want_src=want_src)
    if want_src:
        d, dsrc = out[0].cpu().numpy(), out[1].cpu().numpy()
    else:
        d, dsrc = out.cpu().numpy(), None
    exp = G.export()
    G.close()
    return types.SimpleNamespace(summary=s, A=A, mu=mu, sigma=sig, slack=sl, rf=rf, d_mean=d, d_src=dsrc,
                                 export=exp)


def run_oracle(g, tau=0.0, dslack=None):
    f = oracle.forward(g, NS, tau)
    s = oracle.slack(g, f["A"])
    b = oracle.backward(g, NS, tau, dslack=dslack)
    return f, s, b


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_levelization_bit_exact(cfg):
    g = synth.generate(cfg)
    G = insta.Graph(g)
    e = G.export()
    o = oracle.levelize(g.num_pins, g.arc_from, g.arc_to)
    for k in ("level", "order", "fanin_ptr", "fanin_arc", "fanout_ptr", "fanout_arc"):
        assert np.array_equal(e[k], o[k]), k
    assert G.num_levels == o["num_levels"]


@pytest.mark.parametrize("cfg", ["C1", "C2"])
@pytest.mark.parametrize("schedule", [0, 1, 2, 3])
def test_dyadic_hard_bit_exact(cfg, schedule):
    """sigma = 0 and mu on a 2^-6 grid: fp32 sums are exact, so GPU == oracle bit for bit,
    including tie-breaking (first candidate wins)."""
    g = synth.generate(cfg, dyadic=True)
    r = run_gpu(g, 0.0, schedule)
    f, s, b = run_oracle(g, 0.0)
    assert np.array_equal(r.A, f["A"].astype(np.float32))
    assert np.array_equal(r.slack, s["slack"].astype(np.float32))
    assert np.array_equal(r.rf, s["rf_star"])
    assert r.summary.tns == s["tns"] and r.summary.wns == s["wns"]
    assert r.summary.num_violations == s["num_viol"]
    assert np.array_equal(r.d_mean, b["d_mean"].astype(np.float32))


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_hard_parity(cfg):
    g = synth.generate(cfg)
    r = run_gpu(g, 0.0)
    f, s, b = run_oracle(g, 0.0)
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    assert ft.mean() < 0.01
    assert not tol_ok(r.A, f["A"], ft).any()
    assert not tol_ok(r.mu, f["mu"], ft).any()
    ep_t = ft[g.ep_pin].any(axis=1)
    assert not tol_ok(r.slack, s["slack"], ep_t).any()
    assert r.summary.num_violations == pytest.approx(s["num_viol"], abs=max(1, ep_t.sum()))
    assert r.summary.tns == pytest.approx(s["tns"], rel=1e-5)
    # hard-mode gradients are (negated) path counts: exact away from near-ties
    bad = (r.d_mean != b["d_mean"]) & ~at
    assert not bad.any(), np.argwhere(bad)[:5]
    assert at.mean() < 0.01


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_lse_tau1_parity(cfg):
    g = synth.generate(cfg)
    r = run_gpu(g, 1.0, want_src=True)
    f, s, b = run_oracle(g, 1.0)
    assert not tol_ok(r.A, f["A"]).any()
    assert not tol_ok(r.slack, s["slack"]).any()
    assert r.summary.tns == pytest.approx(s["tns"], rel=1e-5)
    err = np.abs(r.d_mean - b["d_mean"])
    assert (err <= 1e-3 * np.maximum(np.abs(b["d_mean"]), 1.0)).all(), err.max()
    srcmask = np.bincount(g.arc_to, minlength=g.num_pins) == 0
    assert np.abs(r.d_src[srcmask] - b["d_src_mean"][srcmask]).max() <= 1e-3 * max(1, np.abs(b["d_src_mean"]).max())


def test_lse_tau_0p01_normwise_c1():
    """tau = 0.01 ps (the INSTA-Size value): fp32 arrival rounding is a visible
    fraction of tau, so gradients are compared norm-wise."""
    g = synth.generate("C1")
    r = run_gpu(g, 0.01)
    f, s, b = run_oracle(g, 0.01)
    assert not tol_ok(r.A, f["A"]).any()
    rel = np.linalg.norm(r.d_mean - b["d_mean"]) / np.linalg.norm(b["d_mean"])
    assert rel <= 1e-3, rel


def grads_match(x, y, tau):
    """Gradients of two schedules: the sweep (0) accumulates adjoints in 2^-32 fixed point, the
    others sum fp32 per-arc adjoints, so they agree bit for bit where the adjoints are integers
    (hard mode: path counts) and to fp32 summation rounding otherwise."""
    if tau == 0.0:
        return np.array_equal(x, y)
    return bool((np.abs(x - y) <= 1e-5 * np.maximum(np.abs(y), 1.0)).all())


@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_schedules_and_reruns_bit_identical(tau):
    """Forward results are the same bit for bit under every schedule (same merge arithmetic);
    reruns of a schedule are bit-identical in full (deterministic accumulation)."""
    g = synth.generate("C2")
    a = run_gpu(g, tau, 0)
    c = run_gpu(g, tau, 1)
    e = run_gpu(g, tau, 2)
    f = run_gpu(g, tau, 3)
    d = run_gpu(g, tau, 0)
    for x, y in ((a, c), (a, d), (a, e), (a, f)):
        assert np.array_equal(x.A, y.A) and np.array_equal(x.sigma, y.sigma)
        assert np.array_equal(x.slack, y.slack) and x.summary == y.summary
    assert np.array_equal(a.d_mean, d.d_mean) and np.array_equal(a.d_mean, f.d_mean)
    assert np.array_equal(c.d_mean, e.d_mean)
    assert grads_match(a.d_mean, c.d_mean, tau)


def test_custom_endpoint_seed_and_source_gradient():
    g = synth.generate("C1")
    rng = np.random.default_rng(7)
    seed = rng.uniform(-1, 1, g.num_endpoints).astype(np.float32)
    r = run_gpu(g, 1.0, seed=seed, want_src=True)
    _, _, b = run_oracle(g, 1.0, dslack=seed.astype(np.float64))
    assert np.abs(r.d_mean - b["d_mean"]).max() <= 1e-3 * max(1.0, np.abs(b["d_mean"]).max())
    assert np.abs(r.d_src - b["d_src_mean"]).max() <= 1e-3 * max(1.0, np.abs(b["d_src_mean"]).max())


@pytest.mark.parametrize("tau", [0.0, 1.0])
@pytest.mark.parametrize("schedule", [0, 1, 2, 3])
def test_backward_overwrites_poisoned_outputs(tau, schedule):
    """insta_backward fully defines its outputs (include/insta.h): outputs prefilled
    with NaN, at an 8-byte offset (not 16-byte aligned, odd float2 count) so the
    prologue kernel's zero fill covers its unaligned head and tail, give the
    same gradients, bit for bit, as fresh buffers (which the other tests check
    against the oracle)."""
    import torch

    g = synth.generate("C2")
    G = insta.Graph(g)
    G.forward(NS, tau, schedule)
    ref = G.backward().cpu().numpy()
    E = g.num_arcs
    raw = torch.full((2 * E + 2,), float("nan"), dtype=torch.float32, device="cuda")
    out = raw[2:].view(E, 2)   # 8-byte offset
    d = G.backward(out=out).cpu().numpy()
    G.close()
    assert np.isfinite(d).all()                            # every element written (zero or gradient)
    assert np.array_equal(d, ref)
    assert np.isnan(raw[:2].cpu().numpy()).all()          # nothing written before the buffer


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_tiny_dags(seed, tau):
    g = bf.tiny_dag(seed, n_pins=9)
    r = run_gpu(g, tau)
    f, s, b = run_oracle(g, tau)
    ft, at = oracle.tie_taint(g, NS, eps=1e-4, margin=0.05)
    assert not tol_ok(r.A, f["A"], ft if tau == 0 else None).any()
    mask = at if tau == 0 else np.zeros_like(at)
    err = np.abs(r.d_mean - b["d_mean"])
    assert ((err <= 1e-3 * np.maximum(np.abs(b["d_mean"]), 1)) | mask).all()


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("tau", [0.3, 2.0])
def test_lse_sigma_pos_equal_variance_layered(seed, tau):
    """LSE with sigma > 0 on the layered equal-variance DAGs of the oracle pin: the GPU matches the
    oracle and the closed form tau*logsumexp(path means) + N_sigma*sqrt(common variance)."""
    from scipy.special import logsumexp
    g, lvl = bf.layered_equal_variance(seed)
    r = run_gpu(g, tau)
    f, s, b = run_oracle(g, tau)
    assert not tol_ok(r.A, f["A"]).any()
    for (i, rf), ps in bf.enumerate_paths(g).items():
        want = tau * logsumexp(np.array([m for m, _, _ in ps]) / tau) + NS * np.sqrt(1.5 ** 2 + lvl[i] * 4.0)
        assert abs(r.A[i][rf] - want) <= max(1e-4 * abs(want), 1e-3)
    assert (np.abs(r.d_mean - b["d_mean"]) <= 1e-3 * np.maximum(np.abs(b["d_mean"]), 1)).all()


def _star(n_sinks, tau_unate=2, wide=9):
    """One driver with a huge fanout (> 128, the heavy-driver path) and a wide
    (9-input) NON-unate cell: exercises the atomic accumulator and the slow fanin path."""
    rng = np.random.default_rng(n_sinks)
    src, drv = 0, 1
    sinks = np.arange(2, 2 + n_sinks)
    cell_in = sinks[:wide]
    out = 2 + n_sinks
    af = [src] + [drv] * n_sinks + list(cell_in)
    at = [drv] + list(sinks) + [out] * wide
    E = len(af)
    un = np.zeros(E, np.uint8)
    un[1 + n_sinks:] = tau_unate
    mean = rng.uniform(1, 10, (E, 2)).astype(np.float32)
    sig = rng.uniform(0, 1, (E, 2)).astype(np.float32)
    N = out + 1
    eps = np.concatenate([sinks[wide:], [out]]).astype(np.int32)
    rat = np.full((len(eps), 2), 18.0, np.float32)
    sm = np.zeros((N, 2), np.float32)
    ss = np.zeros((N, 2), np.float32)
    ss[0] = 0.5
    return types.SimpleNamespace(num_pins=N, arc_from=np.array(af, np.int32), arc_to=np.array(at, np.int32),
                                 arc_unate=un, arc_class=np.zeros(E, np.uint8), arc_mean=mean, arc_sigma=sig,
                                 src_mean=sm, src_sigma=ss, ep_pin=eps, ep_rat=rat)


@pytest.mark.parametrize("n_sinks", [40, 3000])
@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_heavy_fanout_and_wide_fanin(n_sinks, tau):
    g = _star(n_sinks)
    r = run_gpu(g, tau, want_src=True)
    f, s, b = run_oracle(g, tau)
    assert not tol_ok(r.A, f["A"]).any()
    err = np.abs(r.d_mean - b["d_mean"])
    assert (err <= 1e-3 * np.maximum(np.abs(b["d_mean"]), 1)).all(), err.max()
    assert np.abs(r.d_src - b["d_src_mean"]).max() <= 1e-3 * max(1, np.abs(b["d_src_mean"]).max())
    r1 = run_gpu(g, tau, schedule=1)
    assert grads_match(r.d_mean, r1.d_mean, tau)


def test_degenerate_graphs():
    # no arcs: all pins are sources; endpoints at sources
    g = types.SimpleNamespace(num_pins=3, arc_from=np.zeros(0, np.int32), arc_to=np.zeros(0, np.int32),
                              arc_unate=np.zeros(0, np.uint8), arc_class=None, arc_mean=np.zeros((0, 2), np.float32),
                              arc_sigma=np.zeros((0, 2), np.float32),
                              src_mean=np.array([[1, 2], [3, 4], [5, 6]], np.float32),
                              src_sigma=np.zeros((3, 2), np.float32),
                              ep_pin=np.array([2, 0], np.int32), ep_rat=np.array([[4, 4], [0, 5]], np.float32))
    r = run_gpu(g, 0.0, want_src=True)
    assert list(r.slack) == [-2.0, -1.0]
    assert r.summary.tns == -3.0 and r.summary.num_violations == 2
    assert np.array_equal(r.d_src, np.array([[-1, 0], [0, 0], [0, -1]], np.float32))  # pin 2: F slack -2 < R slack -1
    # no endpoints
    g2 = bf.tiny_dag(1)
    g2.ep_pin = np.zeros(0, np.int32)
    g2.ep_rat = np.zeros((0, 2), np.float32)
    r2 = run_gpu(g2, 0.0)
    assert r2.summary.tns == 0.0 and not r2.d_mean.any()


def test_call_order_errors():
    g = synth.generate("C1")
    G = insta.Graph(g)
    with pytest.raises(insta.InstaError, match="E_STATE"):
        G.backward()
    G.forward()
    G.update_arcs([0], np.ones((1, 2)), np.zeros((1, 2)), incremental=False)
    with pytest.raises(insta.InstaError, match="E_STATE"):
        G.slack()
    with pytest.raises(insta.InstaError, match="E_ARG"):
        G.forward(tau=-1.0)
    G.close()


def test_update_arcs_then_forward_equals_fresh_graph():
    g = synth.generate("C2")
    ids, m, s = synth.sizing_step(g, 0)
    G = insta.Graph(g)
    G.forward()
    G.update_arcs(ids, m, s, incremental=False)
    G.forward()
    A1 = G.arrivals()[0].cpu().numpy()
    d1 = G.backward().cpu().numpy()
    g2 = types.SimpleNamespace(**vars(g))
    g2.arc_mean = g.arc_mean.copy()
    g2.arc_sigma = g.arc_sigma.copy()
    g2.arc_mean[ids] = m
    g2.arc_sigma[ids] = s
    r = run_gpu(g2, 0.0)
    assert np.array_equal(A1, r.A) and np.array_equal(d1, r.d_mean)


@pytest.mark.slow
def test_c4_full_size_parity():
    """15M pins, the bench configuration (persistent kernels, hard mode): levelization
    bit-exact, arrivals/slack within tolerance everywhere outside near-tie taint, TNS."""
    g = synth.generate("C4")
    G = insta.Graph(g)
    summ = G.forward(NS, 0.0)
    e = G.export()
    o = oracle.levelize(g.num_pins, g.arc_from, g.arc_to)
    for k in ("level", "order", "fanin_ptr", "fanin_arc", "fanout_ptr", "fanout_arc"):
        assert np.array_equal(e[k], o[k]), k
    del e, o
    A = G.arrivals()[0].cpu().numpy()
    sl = G.slack()[0].cpu().numpy()
    f = oracle.forward(g, NS, 0.0)
    s = oracle.slack(g, f["A"])
    ft, at = oracle.tie_taint(g, NS, eps=1e-3, margin=0.05)
    assert ft.mean() < 0.01
    assert not tol_ok(A, f["A"], ft).any()
    assert not tol_ok(sl, s["slack"], ft[g.ep_pin].any(axis=1)).any()
    assert summ.tns == pytest.approx(s["tns"], rel=1e-5)
    # gradients: hard mode, exact integers away from near-ties
    d = G.backward().cpu().numpy()
    b = oracle.backward(g, NS, 0.0)
    assert at.mean() < 0.01
    assert not ((d != b["d_mean"]) & ~at).any()
    G.close()


@pytest.mark.slow
def test_c4_full_size_lse_tau1_parity():
    """15M pins, LSE tau = 1 ps (the differentiable mode, Eq 4 / Eq 6): arrivals and slack within
    max(1e-4 |x|, 1e-3 ps) everywhere, TNS, and every arc's gradient within 1e-3 max(|g|, 1) of the oracle
    (no exemptions: the LSE merge has no kinks)."""
    g = synth.generate("C4")
    G = insta.Graph(g)
    summ = G.forward(NS, 1.0)
    A = G.arrivals()[0].cpu().numpy()
    sl = G.slack()[0].cpu().numpy()
    d = G.backward().cpu().numpy()
    G.close()
    f = oracle.forward(g, NS, 1.0)
    s = oracle.slack(g, f["A"])
    assert not tol_ok(A, f["A"]).any()
    assert not tol_ok(sl, s["slack"]).any()
    assert summ.tns == pytest.approx(s["tns"], rel=1e-5)
    del f
    b = oracle.backward(g, NS, 1.0)
    err = np.abs(d - b["d_mean"])
    assert (err <= 1e-3 * np.maximum(np.abs(b["d_mean"]), 1.0)).all(), err.max()


def _fold_shapes(seed=3):
    """Graph shapes that exercise the stage-folded forward (fold.cpp): a
    fanin-1/fanout-1 chain (folds alternate), cells whose inputs are all
    folded with 3, 40 (> 32 arcs: single-lane merge) and 1500 (> the item
    cap: direct path) inputs, non-unate arcs on both sides of a folded pin,
    a folded pin driven by a heavy (> 256 sinks) driver, and an endpoint with
    fanout 1 (never folded)."""
    rng = np.random.default_rng(seed)
    af, at, un = [], [], []
    n = [0]

    def pin():
        n[0] += 1
        return n[0] - 1

    def arc(a, b, u):
        af.append(a)
        at.append(b)
        un.append(u)

    srcs = [pin() for _ in range(8)]
    eps = []
    # chain
    x = srcs[0]
    for k in range(20):
        y = pin()
        arc(x, y, int(rng.integers(0, 3)))
        x = y
    eps.append(x)
    # heavy driver with 300 sinks, each feeding a 3-input cell
    drv = pin()
    arc(srcs[1], drv, 0)
    sinks = [pin() for _ in range(300)]
    for s_ in sinks:
        arc(drv, s_, 0)
    for c in range(100):
        out = pin()
        for s_ in sinks[3 * c:3 * c + 3]:
            arc(s_, out, int(rng.integers(0, 3)))
        eps.append(out)
    # wide cells: inputs are net sinks of random earlier drivers
    for width in (40, 1500):
        out = pin()
        for k in range(width):
            ip = pin()
            arc(int(rng.choice(srcs)), ip, int(rng.integers(0, 3)))
            arc(ip, out, int(rng.integers(0, 3)))
        eps.append(out)
    # an endpoint with one fanin and one fanout: not folded
    e1 = pin()
    arc(srcs[2], e1, 1)
    e2 = pin()
    arc(e1, e2, 2)
    eps += [e1, e2]
    N, E = n[0], len(af)
    return types.SimpleNamespace(
        num_pins=N, arc_from=np.array(af, np.int32), arc_to=np.array(at, np.int32),
        arc_unate=np.array(un, np.uint8), arc_class=np.zeros(E, np.uint8),
        arc_mean=rng.uniform(1, 10, (E, 2)).astype(np.float32),
        arc_sigma=rng.uniform(0, 1, (E, 2)).astype(np.float32),
        src_mean=rng.uniform(0, 5, (N, 2)).astype(np.float32), src_sigma=rng.uniform(0, 1, (N, 2)).astype(np.float32),
        ep_pin=np.array(eps, np.int32), ep_rat=np.full((len(eps), 2), 40.0, np.float32))


@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_stage_folded_shapes(tau):
    g = _fold_shapes()
    a = run_gpu(g, tau, 0, want_src=True)
    c = run_gpu(g, tau, 1, want_src=True)
    e = run_gpu(g, tau, 2, want_src=True)
    f3 = run_gpu(g, tau, 3, want_src=True)
    assert np.array_equal(a.d_mean, f3.d_mean) and np.array_equal(a.A, f3.A)
    for y in (c, e):
        assert np.array_equal(a.A, y.A) and np.array_equal(a.mu, y.mu) and np.array_equal(a.sigma, y.sigma)
        assert grads_match(a.d_mean, y.d_mean, tau) and grads_match(a.d_src, y.d_src, tau)
    assert np.array_equal(c.d_mean, e.d_mean) and np.array_equal(c.d_src, e.d_src)
    f, s, b = run_oracle(g, tau)
    ft, at = oracle.tie_taint(g, NS, eps=1e-4, margin=0.05)
    assert not tol_ok(a.A, f["A"], ft if tau == 0 else None).any()
    mask = at if tau == 0 else np.zeros_like(at)
    err = np.abs(a.d_mean - b["d_mean"])
    assert ((err <= 1e-3 * np.maximum(np.abs(b["d_mean"]), 1)) | mask).all()


def _sigma_case(g, tau):
    G = insta.Graph(g)
    G.forward(NS, tau)
    d0, dsrc0 = (x.cpu().numpy() for x in G.backward(want_src=True))
    d1, ds, dsrc1 = (x.cpu().numpy() for x in G.backward(want_src=True, want_sigma=True))
    G.close()
    # the sigma pass reproduces the mean channel (bit for bit in hard mode; to the
    # fp32-sum vs fixed-point accumulation rounding with tau > 0)
    assert grads_match(d0, d1, tau) and grads_match(dsrc0, dsrc1, tau)
    b = oracle.backward(g, NS, tau)
    mask = oracle.tie_taint(g, NS, eps=1e-4, margin=0.05)[1] if tau == 0 else np.zeros(ds.shape, bool)
    err = np.abs(ds - b["d_sigma"])
    bad = (err > 1e-3 * np.maximum(np.abs(b["d_sigma"]), 1)) & ~mask
    assert not bad.any(), (err[bad].max(), int(bad.sum()))
    assert mask.mean() < 0.01
    return ds, b["d_sigma"]


@pytest.mark.parametrize("cfg", ["C1", "C2"])
@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_sigma_gradient_parity(cfg, tau):
    """dTNS/d(arc sigma) (reading R1) vs the fp64 oracle."""
    ds, ref = _sigma_case(synth.generate(cfg), tau)
    assert np.count_nonzero(ref) > 0


@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_sigma_gradient_shapes(tau):
    """Heavy driver (fixed-point accumulation of both channels), wide non-unate
    fanin, folded-pin shapes and the appendix example (sigma at a zero-sigma arc)."""
    _sigma_case(_star(3000), tau)
    _sigma_case(_fold_shapes(), tau)
    for seed in range(4):
        _sigma_case(bf.tiny_dag(seed, n_pins=9), tau)


@pytest.mark.parametrize("mode", ["hard", "lse_tau1"])
def test_appendix_a_gpu(mode):
    """The hand-worked example (tests/golden/appendix_a.json):
    arrivals, slack, dTNS/dmean and dTNS/dsigma from the GPU path."""
    import json
    import os
    d = json.load(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "appendix_a.json")))
    g = types.SimpleNamespace(
        num_pins=d["num_pins"], arc_from=np.array(d["arc_from"], np.int32), arc_to=np.array(d["arc_to"], np.int32),
        arc_unate=np.array(d["arc_unate"], np.uint8), arc_class=None,
        arc_mean=np.array(d["arc_mean"], np.float32), arc_sigma=np.array(d["arc_sigma"], np.float32),
        src_mean=np.array(d["src_mean"], np.float32), src_sigma=np.array(d["src_sigma"], np.float32),
        ep_pin=np.array(d["ep_pin"], np.int32), ep_rat=np.array(d["ep_rat"], np.float32))
    h = d[mode]
    tau = h.get("tau", 0.0)
    G = insta.Graph(g)
    G.forward(d["n_sigma"], tau)
    A = G.arrivals()[0].cpu().numpy()
    for name, pin in (("A_y", 2), ("A_z", 3), ("A_w", 4)):
        assert np.allclose(A[pin], h[name], atol=1e-3)
    dm, ds = (x.cpu().numpy() for x in G.backward(want_sigma=True))
    G.close()
    want_m = np.zeros((5, 2))
    want_s = np.zeros((5, 2))
    for k, v in h["d_mean_nonzero"].items():
        e, r = map(int, k.split(","))
        want_m[e, r] = v
    for k, v in h["d_sigma_nonzero"].items():
        e, r = map(int, k.split(","))
        want_s[e, r] = v
    assert np.allclose(dm, want_m, atol=1e-3) and np.allclose(ds, want_s, atol=1e-3)


def _wide_level(n_heads, wide_fanin, seed=5):
    """One level of n_heads single-input endpoint heads (more than 1024 per CTA slice: the entry-
    parallel forward reads that slice's topology from global) plus one head with wide_fanin inputs
    (more entries than a slice's shared-memory candidate buffer: the CTA's global buffer)."""
    rng = np.random.default_rng(seed)
    n_src = n_heads + wide_fanin
    N = n_src + n_heads + 1
    src = np.arange(n_src)
    af = np.concatenate([src[:n_heads], src[n_heads:]]).astype(np.int32)
    at = np.concatenate([n_src + np.arange(n_heads), np.full(wide_fanin, N - 1)]).astype(np.int32)
    E = len(af)
    un = rng.integers(0, 3, E).astype(np.uint8)
    mean = rng.uniform(1, 20, (E, 2)).astype(np.float32)
    sig = rng.uniform(0, 2, (E, 2)).astype(np.float32)
    eps = np.arange(n_src, N, dtype=np.int32)
    rat = rng.uniform(40, 60, (len(eps), 2)).astype(np.float32)
    return types.SimpleNamespace(num_pins=N, arc_from=af, arc_to=at, arc_unate=un,
                                 arc_class=np.zeros(E, np.uint8), arc_mean=mean, arc_sigma=sig,
                                 src_mean=rng.uniform(0, 30, (N, 2)).astype(np.float32),
                                 src_sigma=rng.uniform(0, 3, (N, 2)).astype(np.float32), ep_pin=eps, ep_rat=rat)


@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_forward_unstaged_and_global_candidate_paths(tau):
    # 160k heads in one level (1081 per CTA > the 1024-row stage) and a 3000-input head (> 2048
    # candidate slots and > 2560 staged entries): schedule 0 (flow) and 3 (barriers) equal the
    # per-level schedule bit for bit and the oracle within tolerance
    g = _wide_level(160_000, 3000)
    a = run_gpu(g, tau, 0)
    b = run_gpu(g, tau, 3)
    c = run_gpu(g, tau, 1)
    for x in (a, b):
        assert np.array_equal(x.A, c.A) and np.array_equal(x.mu, c.mu) and np.array_equal(x.sigma, c.sigma)
        assert np.array_equal(x.slack, c.slack)
        assert grads_match(x.d_mean, c.d_mean, tau)
    f, s, o = run_oracle(g, tau)
    assert not tol_ok(a.A, f["A"]).any()
    assert abs(a.summary.tns - s["tns"]) <= 1e-5 * abs(s["tns"]) + 1e-3
