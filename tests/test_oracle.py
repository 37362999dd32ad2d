"""Pins for the fp64 CPU oracle (oracle/oracle.c) -- run without a GPU.

Each test checks the oracle against something other than itself: brute-force
path enumeration, networkx / scipy library routines, closed forms, the
hand-worked example (tests/golden/appendix_a.json), central finite
differences, and invariants.  Citations are PAPER.md lines (P:Lnn).
"""
import json
import os
import types

import networkx as nx
import numpy as np
import pytest
from scipy.special import logsumexp

import oracle
from tests import bruteforce as bf
from paper_conf_dac_lugklr25_b200 import synth

HERE = os.path.dirname(os.path.abspath(__file__))
NS = 3.0  # N_sigma = 3.0


def _golden():
    with open(os.path.join(HERE, "golden", "appendix_a.json")) as f:
        d = json.load(f)
    g = types.SimpleNamespace(
        num_pins=d["num_pins"], arc_from=np.array(d["arc_from"], np.int32),
        arc_to=np.array(d["arc_to"], np.int32), arc_unate=np.array(d["arc_unate"], np.uint8),
        arc_mean=np.array(d["arc_mean"], float), arc_sigma=np.array(d["arc_sigma"], float),
        src_mean=np.array(d["src_mean"], float), src_sigma=np.array(d["src_sigma"], float),
        ep_pin=np.array(d["ep_pin"], np.int32), ep_rat=np.array(d["ep_rat"], float))
    return d, g


# --------------------------------------------------------------------------- levelization
@pytest.mark.parametrize("seed", range(20))
def test_levelize_matches_networkx_generations(seed):
    """O2: ASAP levels == networkx.topological_generations; canonical order by (level, id)."""
    g = bf.tiny_dag(seed, n_pins=9)
    lv = oracle.levelize(g.num_pins, g.arc_from, g.arc_to)
    G = nx.MultiDiGraph()
    G.add_nodes_from(range(g.num_pins))
    G.add_edges_from(zip(g.arc_from.tolist(), g.arc_to.tolist()))
    gens = list(nx.topological_generations(G))
    assert lv["num_levels"] == len(gens)
    for l, gen in enumerate(gens):
        for p in gen:
            assert lv["level"][p] == l
    expect_order = sorted(range(g.num_pins), key=lambda p: (lv["level"][p], p))
    assert list(lv["order"]) == expect_order


def test_levelize_c2_invariants_and_csr():
    g = synth.generate("C2")
    lv = oracle.levelize(g.num_pins, g.arc_from, g.arc_to)
    level = lv["level"]
    assert np.all(level[g.arc_to] > level[g.arc_from])
    # every non-source pin has a fanin at exactly level-1 (ASAP / longest path)
    best = np.full(g.num_pins, -1)
    np.maximum.at(best, g.arc_to, level[g.arc_from])
    has_in = np.bincount(g.arc_to, minlength=g.num_pins) > 0
    assert np.all(best[has_in] == level[has_in] - 1)
    assert np.all(level[~has_in] == 0)
    # CSR rows: fanin row k holds exactly the arcs into order[k], ascending
    pos = np.empty(g.num_pins, np.int64)
    pos[lv["order"]] = np.arange(g.num_pins)
    fp, fa = lv["fanin_ptr"], lv["fanin_arc"]
    assert fp[-1] == g.num_arcs
    assert np.all(pos[g.arc_to[fa]] == np.repeat(np.arange(g.num_pins), np.diff(fp)))
    row = np.repeat(np.arange(g.num_pins), np.diff(fp))
    assert np.all((np.diff(fa) > 0) | (np.diff(row) != 0))
    op, oa = lv["fanout_ptr"], lv["fanout_arc"]
    assert np.all(pos[g.arc_from[oa]] == np.repeat(np.arange(g.num_pins), np.diff(op)))
    G = nx.DiGraph()
    G.add_nodes_from(range(g.num_pins))
    G.add_edges_from(zip(g.arc_from.tolist(), g.arc_to.tolist()))
    assert lv["num_levels"] == nx.dag_longest_path_length(G) + 1


def test_levelize_detects_cycle():
    with pytest.raises(oracle.OracleError, match="cycle"):
        oracle.levelize(3, np.array([0, 1, 2]), np.array([1, 2, 0]))
    with pytest.raises(oracle.OracleError, match="cycle"):
        oracle.levelize(2, np.array([1]), np.array([1]))   # self loop


# --------------------------------------------------------------------------- hard forward
@pytest.mark.parametrize("seed", range(25))
def test_hard_sigma0_equals_bruteforce_max_path(seed):
    """sigma == 0, K = 1 (Alg 1/2): the corner arrival is the max over all timing paths, exactly."""
    g = bf.tiny_dag(seed, sigma0=True, dyadic=True)
    f = oracle.forward(g, NS, 0.0)
    paths = bf.enumerate_paths(g)
    for (i, rf), ps in paths.items():
        assert f["A"][i][rf] == max(m for m, _, _ in ps)


def test_hard_sigma0_equals_networkx_longest_path_on_expanded_graph():
    """C1 dyadic: A at each endpoint == networkx.dag_longest_path_length on the (pin, rf) graph."""
    g = synth.generate("C1", dyadic=True)
    f = oracle.forward(g, NS, 0.0)
    G = nx.DiGraph()
    src = "S"
    has_in = np.bincount(g.arc_to, minlength=g.num_pins) > 0
    for p in np.nonzero(~has_in)[0]:
        for rf in (0, 1):
            G.add_edge(src, (int(p), rf), weight=float(g.src_mean[p][rf]))
    for e in range(g.num_arcs):
        j, i = int(g.arc_from[e]), int(g.arc_to[e])
        for rf in (0, 1):
            for s in bf.source_transitions(rf, int(g.arc_unate[e])):
                G.add_edge((j, s), (i, rf), weight=float(g.arc_mean[e][rf]))
    dist = {src: 0.0}
    for v in nx.topological_sort(G):
        if v == src:
            continue
        dist[v] = max(dist[u] + G[u][v]["weight"] for u in G.predecessors(v))
    for k in g.ep_pin[:50]:
        for rf in (0, 1):
            assert f["A"][k][rf] == dist[(int(k), rf)]
    # networkx's own routine on the whole expanded graph = the max over all pins
    assert nx.dag_longest_path_length(G) == pytest.approx(f["A"].max(), abs=0)


@pytest.mark.parametrize("seed", range(25))
def test_hard_sigma_pos_traced_path_identity_and_upper_bound(seed):
    """sigma > 0: A equals the corner of its traced critical path exactly (Eq 1-3), and is <= the
    brute-force max path corner (block-based propagation keeps one distribution per pin)."""
    g = bf.tiny_dag(seed)
    f = oracle.forward(g, NS, 0.0)
    paths = bf.enumerate_paths(g)
    arcs_m, arcs_s = np.asarray(g.arc_mean), np.asarray(g.arc_sigma)
    for (i, rf), ps in paths.items():
        sp, r, hops = bf.trace_critical(g, f["win_arc"], f["win_s"], i, rf)
        m = g.src_mean[sp][r] + sum(arcs_m[e][x] for e, x in hops)
        v = g.src_sigma[sp][r] ** 2 + sum(arcs_s[e][x] ** 2 for e, x in hops)
        assert f["A"][i][rf] == pytest.approx(bf.corner(m, v, NS), abs=1e-9)
        assert f["A"][i][rf] <= max(bf.corner(pm, pv, NS) for pm, pv, _ in ps) + 1e-9
        assert f["mu"][i][rf] == pytest.approx(m, abs=1e-9)


def test_hard_first_candidate_wins_ties():
    """Strict '>' (Alg 2 l.4): among equal corners the earliest candidate (lowest arc id,
    then s = rf before ~rf) wins."""
    g = types.SimpleNamespace(
        num_pins=3, arc_from=np.array([1, 0], np.int32), arc_to=np.array([2, 2], np.int32),
        arc_unate=np.array([0, 2], np.uint8), arc_mean=np.array([[5.0, 5.0], [5.0, 5.0]]),
        arc_sigma=np.zeros((2, 2)), src_mean=np.zeros((3, 2)), src_sigma=np.zeros((3, 2)),
        ep_pin=np.array([2], np.int32), ep_rat=np.array([[1.0, 1.0]]))
    f = oracle.forward(g, NS, 0.0)
    assert f["win_arc"][2][0] == 0 and f["win_s"][2][0] == 0
    assert f["win_arc"][2][1] == 0 and f["win_s"][2][1] == 1


# --------------------------------------------------------------------------- LSE forward
@pytest.mark.parametrize("seed", range(20))
@pytest.mark.parametrize("tau", [0.01, 0.5, 3.0])
def test_lse_sigma0_equals_logsumexp_over_all_paths(seed, tau):
    """Block LSE (Eq 4) with sigma == 0 composes to tau*logsumexp of all path sums (scipy)."""
    g = bf.tiny_dag(seed, sigma0=True)
    f = oracle.forward(g, NS, tau)
    for (i, rf), ps in bf.enumerate_paths(g).items():
        want = tau * logsumexp(np.array([m for m, _, _ in ps]) / tau)
        assert f["A"][i][rf] == pytest.approx(want, rel=1e-12, abs=1e-9)


def _fan(n_in, means, tau, unate=0):
    n = n_in + 1
    return types.SimpleNamespace(
        num_pins=n, arc_from=np.arange(n_in, dtype=np.int32), arc_to=np.full(n_in, n_in, np.int32),
        arc_unate=np.full(n_in, unate, np.uint8), arc_mean=np.array([[m, m] for m in means], float),
        arc_sigma=np.zeros((n_in, 2)), src_mean=np.zeros((n, 2)), src_sigma=np.zeros((n, 2)),
        ep_pin=np.array([n_in], np.int32), ep_rat=np.array([[0.0, 0.0]]))


@pytest.mark.parametrize("n", [1, 2, 3, 7])
def test_lse_closed_form_equal_inputs(n):
    """Eq 4: n equal arrivals x -> x + tau*ln(n); Eq 6: each weight 1/n."""
    tau = 0.7
    g = _fan(n, [4.0] * n, tau)
    assert oracle.forward(g, NS, tau)["A"][n][0] == pytest.approx(4.0 + tau * np.log(n), abs=1e-12)
    b = oracle.backward(g, NS, tau, dslack=np.array([1.0]))
    assert np.allclose(b["d_mean"][:, 0], -1.0 / n, atol=1e-12)


def test_lse_closed_form_two_inputs_and_limit():
    """Two inputs Delta apart: max + tau*ln(1 + exp(-Delta/tau)); tau -> 0 gives the max (Eq 5)."""
    for tau in (0.05, 1.0, 4.0):
        g = _fan(2, [10.0, 7.5], tau)
        want = 10.0 + tau * np.log1p(np.exp(-2.5 / tau))
        assert oracle.forward(g, NS, tau)["A"][2][0] == pytest.approx(want, abs=1e-12)
    g = bf.tiny_dag(3)
    hard = oracle.forward(g, NS, 0.0)["A"]
    soft = oracle.forward(g, NS, 1e-6)["A"]
    assert np.allclose(hard, soft, atol=1e-4)
    # bounds: max <= LSE <= max + tau*ln(#candidates)
    lse = oracle.forward(g, NS, 0.5)["A"]
    assert np.all(lse >= hard - 1e-12)


# --------------------------------------------------------------------------- slack
def test_slack_closed_forms():
    """Slack = RAT - A, min over rf, tie -> R; slack == 0 is not a violation; TNS sums negatives."""
    g = types.SimpleNamespace(
        num_pins=4, arc_from=np.array([], np.int32), arc_to=np.array([], np.int32),
        arc_unate=np.array([], np.uint8), arc_mean=np.zeros((0, 2)), arc_sigma=np.zeros((0, 2)),
        src_mean=np.array([[1.0, 2.0], [5.0, 5.0], [0.0, 0.0], [3.0, 1.0]]), src_sigma=np.zeros((4, 2)),
        ep_pin=np.array([0, 1, 2, 3], np.int32),
        ep_rat=np.array([[0.0, 10.0], [4.0, 4.0], [0.0, 0.0], [10.0, 10.0]]))
    A = oracle.forward(g, NS, 0.0)["A"]
    s = oracle.slack(g, A)
    assert list(s["slack"]) == [-1.0, -1.0, 0.0, 7.0]
    assert list(s["rf_star"]) == [0, 0, 0, 0]
    assert s["tns"] == -2.0 and s["wns"] == -1.0 and s["num_viol"] == 2
    g.ep_rat = np.array([[50.0, 50.0]] * 4)
    s = oracle.slack(g, oracle.forward(g, NS, 0.0)["A"])
    assert s["tns"] == 0.0 and s["wns"] == 0.0 and s["num_viol"] == 0


# --------------------------------------------------------------------------- hand-worked example
def test_appendix_a_hard():
    d, g = _golden()
    h = d["hard"]
    f = oracle.forward(g, d["n_sigma"], 0.0)
    assert list(oracle.levelize(5, g.arc_from, g.arc_to)["level"]) == d["levels"]
    for name, pin in (("A_y", 2), ("A_z", 3), ("A_w", 4)):
        assert f["A"][pin] == pytest.approx(h[name], abs=2e-6)
    assert f["mu"][3] == pytest.approx(h["mu_z"], abs=2e-6)
    assert f["sigma"][4] == pytest.approx(h["sigma_w"], abs=2e-6)
    s = oracle.slack(g, f["A"])
    assert s["slack"] == pytest.approx(h["slack"], abs=2e-6)
    assert s["tns"] == pytest.approx(h["tns"], abs=2e-6) and s["num_viol"] == h["num_viol"]
    b = oracle.backward(g, d["n_sigma"], 0.0)
    want_m = np.zeros((5, 2)); want_s = np.zeros((5, 2))
    for k, v in h["d_mean_nonzero"].items():
        e, r = map(int, k.split(",")); want_m[e, r] = v
    for k, v in h["d_sigma_nonzero"].items():
        e, r = map(int, k.split(",")); want_s[e, r] = v
    assert np.allclose(b["d_mean"], want_m, atol=2e-6)
    assert np.allclose(b["d_sigma"], want_s, atol=2e-6)
    assert b["d_src_mean"][1][0] == pytest.approx(h["d_src_mean_b_R"])


def test_appendix_a_lse():
    d, g = _golden()
    h = d["lse_tau1"]
    f = oracle.forward(g, d["n_sigma"], h["tau"])
    for name, pin in (("A_y", 2), ("A_z", 3), ("A_w", 4)):
        assert f["A"][pin] == pytest.approx(h[name], abs=2e-6)
    s = oracle.slack(g, f["A"])
    assert s["slack"] == pytest.approx(h["slack"], abs=2e-6)
    b = oracle.backward(g, d["n_sigma"], h["tau"])
    for k, v in h["d_mean_nonzero"].items():
        e, r = map(int, k.split(",")); assert b["d_mean"][e, r] == pytest.approx(v, abs=2e-6)
    for k, v in h["d_sigma_nonzero"].items():
        e, r = map(int, k.split(",")); assert b["d_sigma"][e, r] == pytest.approx(v, abs=2e-6)
    assert b["d_src_mean"].sum() == pytest.approx(-1.0, abs=1e-12)


# --------------------------------------------------------------------------- gradients
def _tns(g, tau, **over):
    gg = types.SimpleNamespace(**{**vars(g), **over})
    return oracle.slack(gg, oracle.forward(gg, NS, tau)["A"])["tns"]


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("tau", [0.0, 1.0])
def test_backward_matches_central_finite_differences(seed, tau):
    """dTNS/d(arc mean, arc sigma, source mean, source sigma) vs central differences of forward."""
    g = bf.tiny_dag(seed, n_pins=8)
    g.ep_rat = np.full((len(g.ep_pin), 2), 25.0)
    b = oracle.backward(g, NS, tau)
    h = 1e-6
    checked = 0
    for name, grad in (("arc_mean", b["d_mean"]), ("arc_sigma", b["d_sigma"]),
                       ("src_mean", b["d_src_mean"]), ("src_sigma", b["d_src_sigma"])):
        base = np.asarray(getattr(g, name), float)
        for idx in np.ndindex(base.shape):
            if name.startswith("arc_sigma") and base[idx] < 10 * h:
                continue
            up = base.copy(); up[idx] += h
            dn = base.copy(); dn[idx] -= h
            tu, td = _tns(g, tau, **{name: up}), _tns(g, tau, **{name: dn})
            t0 = _tns(g, tau)
            fd = (tu - td) / (2 * h)
            if tau == 0.0 and abs((tu - t0) - (t0 - td)) > 1e-7:
                continue   # a kink (tie / slack sign change) inside [-h, h]
            assert grad[idx] == pytest.approx(fd, abs=1e-5), (name, idx)
            checked += 1
    assert checked > 10


@pytest.mark.parametrize("seed", range(15))
def test_lse_sigma0_gradient_is_gibbs_path_marginal(seed):
    """sigma == 0 LSE: dA_ep/dmu_e[rf] = sum over paths through (e, rf) of softmax(path/tau)."""
    tau = 0.8
    g = bf.tiny_dag(seed, sigma0=True)
    paths = bf.enumerate_paths(g)
    f = oracle.forward(g, NS, tau)
    s = oracle.slack(g, f["A"])
    for k in range(len(g.ep_pin)):
        dsl = np.zeros(len(g.ep_pin)); dsl[k] = 1.0
        b = oracle.backward(g, NS, tau, dslack=dsl)
        pin, rf = int(g.ep_pin[k]), int(s["rf_star"][k])
        ps = paths[(pin, rf)]
        w = np.exp(np.array([m for m, _, _ in ps]) / tau - logsumexp(np.array([m for m, _, _ in ps]) / tau))
        want = np.zeros((g.num_arcs if hasattr(g, "num_arcs") else len(g.arc_from), 2))
        for wi, (_, _, hops) in zip(w, ps):
            for e, r in hops:
                want[e, r] += wi
        assert np.allclose(-b["d_mean"], want, atol=1e-10)


@pytest.mark.parametrize("seed", range(10))
@pytest.mark.parametrize("tau", [0.3, 2.0])
def test_lse_sigma_pos_equal_variance_closed_form(seed, tau):
    """LSE (Eq 4) with sigma > 0 where every candidate of a pin has the same sigma_c (Eq 2): the
    merged corner is tau*logsumexp over all paths of the path mean sums plus N_sigma*sqrt of the
    common path variance (Eq 1-3), whichever candidate's sigma the merge keeps (so this pins the
    Eq 1-4 bookkeeping of the sigma > 0 LSE merge independently of reading R1); dA/dmu_e is the
    softmax path marginal (Eq 6) since the sigma term is a constant offset."""
    s0, sa = 1.5, 2.0
    g, lvl = bf.layered_equal_variance(seed, s0=s0, sa=sa)
    paths = bf.enumerate_paths(g)
    f = oracle.forward(g, NS, tau)
    for (i, rf), ps in paths.items():
        means = np.array([m for m, _, _ in ps])
        assert np.allclose([v for _, v, _ in ps], s0 ** 2 + lvl[i] * sa ** 2)   # the premise
        want = tau * logsumexp(means / tau) + NS * np.sqrt(s0 ** 2 + lvl[i] * sa ** 2)
        assert f["A"][i][rf] == pytest.approx(want, rel=1e-12, abs=1e-9)
    s = oracle.slack(g, f["A"])
    for k in range(len(g.ep_pin)):
        dsl = np.zeros(len(g.ep_pin)); dsl[k] = 1.0
        b = oracle.backward(g, NS, tau, dslack=dsl)
        ps = paths[(int(g.ep_pin[k]), int(s["rf_star"][k]))]
        means = np.array([m for m, _, _ in ps])
        w = np.exp(means / tau - logsumexp(means / tau))
        want = np.zeros((len(g.arc_from), 2))
        for wi, (_, _, hops) in zip(w, ps):
            for e, r in hops:
                want[e, r] += wi
        assert np.allclose(-b["d_mean"], want, atol=1e-10)


@pytest.mark.parametrize("seed", range(15))
def test_hard_gradient_counts_violating_critical_paths(seed):
    """Hard mode: dTNS/dmu_e[rf] = -(# violating endpoints whose traced critical path uses (e, rf))."""
    g = bf.tiny_dag(seed, n_pins=9)
    g.ep_rat = np.full((len(g.ep_pin), 2), 30.0)
    f = oracle.forward(g, NS, 0.0)
    s = oracle.slack(g, f["A"])
    want = np.zeros((len(g.arc_from), 2))
    for k, pin in enumerate(g.ep_pin):
        if s["slack"][k] < 0:
            _, _, hops = bf.trace_critical(g, f["win_arc"], f["win_s"], int(pin), int(s["rf_star"][k]))
            for e, r in hops:
                want[e, r] -= 1
    b = oracle.backward(g, NS, 0.0)
    assert np.array_equal(b["d_mean"], want)


@pytest.mark.parametrize("tau", [0.0, 0.01, 1.0])
def test_gradient_conservation_c1(tau):
    """Weights sum to 1 per merge: sum over sources of Abar = -#violations (TNS seeds), and
    sum of arc mean-gradients = sum of Abar over non-source pins."""
    g = synth.generate("C1")
    s = oracle.slack(g, oracle.forward(g, NS, tau)["A"])
    b = oracle.backward(g, NS, tau)
    has_in = np.bincount(g.arc_to, minlength=g.num_pins) > 0
    assert b["d_src_mean"].sum() == pytest.approx(-s["num_viol"], rel=1e-9)
    assert b["d_mean"].sum() == pytest.approx(b["abar"][has_in].sum(), rel=1e-9)
    assert np.all(b["d_mean"] <= 1e-15)   # dTNS/dmu <= 0


# --------------------------------------------------------------------------- validation
def test_validation_rejects_bad_inputs():
    g = bf.tiny_dag(1)
    assert oracle.validate(g) == 0
    for field, bad in (("arc_sigma", -1.0), ("arc_mean", np.nan), ("arc_mean", np.inf)):
        x = np.array(getattr(g, field), float); x[0, 0] = bad
        assert oracle.validate(types.SimpleNamespace(**{**vars(g), field: x})) == 1
    assert oracle.validate(g, n_sigma=-1.0) == 1
    assert oracle.validate(g, tau=-0.1) == 1
    dup = types.SimpleNamespace(**{**vars(g), "ep_pin": np.array([0, 0], np.int32),
                                   "ep_rat": np.zeros((2, 2))})
    assert oracle.validate(dup) == 1


def test_openmp_build_matches_serial():
    """The all-core oracle build (OpenMP, pins of a level in parallel; bench cpu_baseline) computes the
    same forward bit for bit and the same backward to rounding (atomic pushes reorder sums)."""
    from paper_conf_dac_lugklr25_b200 import synth
    g = synth.generate("C1")
    for tau in (0.0, 1.0):
        a = oracle.forward(g, 3.0, tau)
        b = oracle.forward(g, 3.0, tau, omp=True)
        assert np.array_equal(a["A"], b["A"]) and np.array_equal(a["win_arc"], b["win_arc"])
        da = oracle.backward(g, 3.0, tau)["d_mean"]
        db = oracle.backward(g, 3.0, tau, omp=True)["d_mean"]
        assert np.allclose(da, db, rtol=1e-12, atol=1e-12)
