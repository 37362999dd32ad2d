"""Pins for the Top-K unique-startpoint oracle -- no GPU.

orc_topk_forward follows Alg 1 and Alg 2 literally;
orc_topk_slack is the CPPR slack of P:L109/L119.  Each test checks them against
something other than themselves:

* K = 1 reduces to the K = 1 hard merge (orc_forward, itself pinned by brute
  force in test_oracle.py), value for value, and its startpoint is the source
  of the traced critical path;
* sigma = 0: the queue at (pin, rf) is the top-K over startpoints of the
  per-startpoint longest path (brute-force path enumeration) -- the Top-K
  problem decomposes when Eq 3 is additive;
* K >= #startpoints, sigma > 0: a startpoint's entry equals the K = 1 hard
  propagation on the graph with every other startpoint removed (each unique-SP
  queue entry is that startpoint's own block-based arrival);
* CPPR slack with sigma = 0 and a full RAT table: min over startpoints of
  RAT(ep, sp) - longest path(sp -> ep), brute force;
* the hand-worked K = 2 example (tests/golden/topk_cppr_appendix_a.json).
"""
import json
import os
import types

import numpy as np
import pytest

import oracle
from tests import bruteforce as bf
from paper_conf_dac_lugklr25_b200 import synth

HERE = os.path.dirname(os.path.abspath(__file__))
NS = 3.0


def _sources(g):
    indeg = np.bincount(np.asarray(g.arc_to), minlength=g.num_pins)
    return np.nonzero(indeg == 0)[0]


def _paths_by_sp(g):
    """(pin, rf) -> {sp: [(mean_sum, var_sum)]} by explicit enumeration (Eq 1-2)."""
    n = g.num_pins
    fanin = [[] for _ in range(n)]
    for e in range(len(g.arc_from)):
        fanin[int(g.arc_to[e])].append(e)
    memo = {}

    def rec(i, rf):
        if (i, rf) in memo:
            return memo[(i, rf)]
        if not fanin[i]:
            out = {i: [(float(g.src_mean[i][rf]), float(g.src_sigma[i][rf]) ** 2)]}
        else:
            out = {}
            for e in fanin[i]:
                j = int(g.arc_from[e])
                for s in bf.source_transitions(rf, int(g.arc_unate[e])):
                    for sp, lst in rec(j, s).items():
                        out.setdefault(sp, []).extend(
                            (m + float(g.arc_mean[e][rf]), v + float(g.arc_sigma[e][rf]) ** 2) for m, v in lst)
        memo[(i, rf)] = out
        return out

    return {(i, rf): rec(i, rf) for i in range(n) for rf in (0, 1)}


def _queue(q, i, rf):
    return [(int(q["sp"][i, rf, k]), float(q["A"][i, rf, k])) for k in range(q["A"].shape[2]) if q["sp"][i, rf, k] >= 0]


# --------------------------------------------------------------------------- structure
@pytest.mark.parametrize("seed", range(12))
def test_topk_queues_sorted_unique(seed):
    """Alg 2 invariants: every queue is descending in A, startpoints are unique, empties trail."""
    g = bf.tiny_dag(seed, n_pins=9, p_edge=0.4)
    for K in (1, 2, 3, 5):
        q = oracle.topk_forward(g, NS, K)
        for i in range(g.num_pins):
            for rf in (0, 1):
                sp = q["sp"][i, rf]
                A = q["A"][i, rf]
                n = int((sp >= 0).sum())
                assert (sp[:n] >= 0).all() and (sp[n:] < 0).all()
                assert len(set(sp[:n].tolist())) == n
                assert (np.diff(A[:n]) <= 0).all()
                assert np.isneginf(A[n:]).all()


# --------------------------------------------------------------------------- K = 1
@pytest.mark.parametrize("seed", range(12))
def test_topk_k1_is_hard_forward(seed):
    """K = 1: Alg 2 keeps the strict-'>' maximum, i.e. the K = 1 merge of orc_forward, bit for bit;
    the stored startpoint is the source of the traced critical path."""
    g = bf.tiny_dag(seed, n_pins=9, p_edge=0.4)
    q = oracle.topk_forward(g, NS, 1)
    f = oracle.forward(g, NS, 0.0)
    assert np.array_equal(q["A"][:, :, 0], f["A"])
    assert np.array_equal(q["mu"][:, :, 0], f["mu"])
    assert np.array_equal(q["sigma"][:, :, 0], f["sigma"])
    for i in range(g.num_pins):
        for rf in (0, 1):
            src, _, _ = bf.trace_critical(g, f["win_arc"], f["win_s"], i, rf)
            assert q["sp"][i, rf, 0] == src


def test_topk_k1_is_hard_forward_c1():
    g = synth.generate("C1")
    q = oracle.topk_forward(g, NS, 1)
    f = oracle.forward(g, NS, 0.0)
    assert np.array_equal(q["A"][:, :, 0], f["A"])
    assert np.array_equal(q["sigma"][:, :, 0], f["sigma"])


# --------------------------------------------------------------------------- sigma = 0: decomposition
@pytest.mark.parametrize("seed", range(16))
def test_topk_sigma0_is_topk_of_per_startpoint_longest_paths(seed):
    """sigma = 0: queue(pin, rf) = the K largest per-startpoint longest-path arrivals (brute force)."""
    g = bf.tiny_dag(seed, n_pins=9, p_edge=0.45, sigma0=True)
    paths = _paths_by_sp(g)
    for K in (1, 2, 3, 9):
        q = oracle.topk_forward(g, NS, K)
        for (i, rf), by_sp in paths.items():
            best = sorted(((max(m for m, _ in lst), sp) for sp, lst in by_sp.items()), key=lambda x: -x[0])[:K]
            got = _queue(q, i, rf)
            assert len(got) == len(best)
            assert [a for _, a in got] == pytest.approx([a for a, _ in best], abs=1e-12)
            # the startpoints match wherever the value is not tied with the next one
            vals = [a for a, _ in best]
            for k, (a, sp) in enumerate(best):
                tied = any(abs(a - v) < 1e-12 for m, v in enumerate(vals) if m != k) or \
                    (k == len(best) - 1 and any(abs(a - max(mm for mm, _ in lst)) < 1e-12
                                                 for s2, lst in by_sp.items() if s2 != sp))
                if not tied:
                    assert got[k][0] == sp


# --------------------------------------------------------------------------- sigma > 0: per-startpoint hard propagation
def _restrict_to_source(g, x):
    """The graph with every startpoint but x removed: arcs out of pins unreachable from x are dropped."""
    n = g.num_pins
    reach = np.zeros(n, bool)
    reach[x] = True
    order = oracle.levelize(n, g.arc_from, g.arc_to)["order"]
    pos = np.empty(n, np.int64)
    pos[order] = np.arange(n)
    for e in np.argsort(pos[np.asarray(g.arc_from)], kind="stable"):
        if reach[g.arc_from[e]]:
            reach[g.arc_to[e]] = True
    keep = reach[np.asarray(g.arc_from)]
    h = types.SimpleNamespace(**vars(g))
    h.arc_from, h.arc_to = g.arc_from[keep], g.arc_to[keep]
    h.arc_unate, h.arc_mean, h.arc_sigma = g.arc_unate[keep], g.arc_mean[keep], g.arc_sigma[keep]
    return h, reach


@pytest.mark.parametrize("seed", range(16))
def test_topk_full_queue_is_per_startpoint_hard_propagation(seed):
    """K >= #startpoints, sigma > 0: the entry of startpoint x at (pin, rf) equals the K = 1 hard
    arrival of (pin, rf) when x is the only startpoint (orc_forward on the restricted graph)."""
    g = bf.tiny_dag(seed, n_pins=9, p_edge=0.45)
    srcs = _sources(g)
    q = oracle.topk_forward(g, NS, len(srcs))
    for x in srcs:
        h, reach = _restrict_to_source(g, int(x))
        f = oracle.forward(h, NS, 0.0)
        for i in np.nonzero(reach)[0]:
            for rf in (0, 1):
                k = np.nonzero(q["sp"][i, rf] == x)[0]
                assert k.size == 1, (i, rf, x)
                k = int(k[0])
                assert q["A"][i, rf, k] == f["A"][i, rf]
                assert q["mu"][i, rf, k] == f["mu"][i, rf]
                assert q["sigma"][i, rf, k] == f["sigma"][i, rf]
        # startpoints that do not reach a pin never appear in its queue
        for i in np.nonzero(~reach)[0]:
            assert not (q["sp"][i] == x).any()


# --------------------------------------------------------------------------- CPPR slack
@pytest.mark.parametrize("seed", range(12))
def test_cppr_slack_sigma0_brute_force(seed):
    """CPPR slack, sigma = 0, K >= #startpoints: min over startpoints reaching the
    endpoint of RAT(ep, sp) - longest path(sp -> ep), with RAT(ep, sp) from the table or the default."""
    g = bf.tiny_dag(seed, n_pins=9, p_edge=0.45, sigma0=True, n_ep=4)
    srcs = _sources(g)
    rng = np.random.default_rng(seed + 77)
    P = len(g.ep_pin)
    ptr, sps, rats = [0], [], []
    for e in range(P):
        chosen = sorted(rng.choice(srcs, size=min(2, len(srcs)), replace=False).tolist())
        for s in chosen:
            sps.append(s)
            rats.append(g.ep_rat[e] + rng.uniform(0, 8, 2))
        ptr.append(len(sps))
    table = (np.array(ptr, np.int32), np.array(sps, np.int32), np.array(rats).reshape(-1, 2))
    q = oracle.topk_forward(g, NS, len(srcs))
    o = oracle.topk_slack(g, q, table)
    paths = _paths_by_sp(g)
    tns = 0.0
    for e in range(P):
        p = int(g.ep_pin[e])
        best = np.inf
        for rf in (0, 1):
            for sp, lst in paths[(p, rf)].items():
                rat = g.ep_rat[e][rf]
                row = list(range(ptr[e], ptr[e + 1]))
                for m in row:
                    if sps[m] == sp:
                        rat = rats[m][rf]
                best = min(best, rat - max(m_ for m_, _ in lst))
        assert o["slack"][e] == pytest.approx(best, abs=1e-9)
        tns += min(0.0, best)
    assert o["tns"] == pytest.approx(tns, abs=1e-9)


def test_cppr_slack_without_table_is_plain_slack_at_k1():
    """No RAT table, K = 1: CPPR slack is orc_slack on the hard arrivals."""
    g = synth.generate("C1")
    q = oracle.topk_forward(g, NS, 1)
    o = oracle.topk_slack(g, q, None)
    f = oracle.forward(g, NS, 0.0)
    s = oracle.slack(g, f["A"])
    assert np.array_equal(o["slack"], s["slack"])
    assert np.array_equal(o["rf_star"], s["rf_star"])
    assert o["tns"] == s["tns"] and o["num_viol"] == s["num_viol"]


# --------------------------------------------------------------------------- hand-worked example
def test_topk_cppr_appendix_a_golden():
    """K = 2 on the Appendix A graph: queues (incl. the in-place update + re-bubble at w) and CPPR slack."""
    with open(os.path.join(HERE, "golden", "appendix_a.json")) as f:
        d = json.load(f)
    with open(os.path.join(HERE, "golden", "topk_cppr_appendix_a.json")) as f:
        t = json.load(f)
    g = types.SimpleNamespace(
        num_pins=d["num_pins"], arc_from=np.array(d["arc_from"], np.int32),
        arc_to=np.array(d["arc_to"], np.int32), arc_unate=np.array(d["arc_unate"], np.uint8),
        arc_mean=np.array(d["arc_mean"], float), arc_sigma=np.array(d["arc_sigma"], float),
        src_mean=np.array(d["src_mean"], float), src_sigma=np.array(d["src_sigma"], float),
        ep_pin=np.array(d["ep_pin"], np.int32), ep_rat=np.array(d["ep_rat"], float))
    q = oracle.topk_forward(g, NS, t["K"])
    pin = {"y": 2, "z": 3, "w": 4}
    for name, rfs in t["queues"].items():
        for rfn, entries in rfs.items():
            rf = 0 if rfn == "R" else 1
            for k, (sp, mu, sig, A) in enumerate(entries):
                i = pin[name]
                assert q["sp"][i, rf, k] == sp, (name, rfn, k)
                assert q["mu"][i, rf, k] == pytest.approx(mu, abs=2e-6)
                assert q["sigma"][i, rf, k] == pytest.approx(sig, abs=2e-6)
                assert q["A"][i, rf, k] == pytest.approx(A, abs=2e-6)
    rt = t["rat_table"]
    o = oracle.topk_slack(g, q, (np.array(rt["ptr"]), np.array(rt["sp"]), np.array(rt["rat"], float)))
    assert o["slack"] == pytest.approx(t["slack"], abs=2e-6)
    assert list(o["rf_star"]) == t["rf_star"]
    assert list(o["k_star"]) == t["k_star"]
    assert list(o["sp_star"]) == t["sp_star"]
    assert o["tns"] == pytest.approx(t["tns"], abs=2e-6)
    assert o["num_viol"] == t["num_violations"]


def test_cppr_rat_table_generator_structure():
    """The synthetic CPPR table only names startpoints in each endpoint's fanin cone, sorted, unique."""
    g = synth.generate("C1")
    ptr, sp, rat = synth.cppr_rat_table(g)
    srcs = set(_sources(g).tolist())
    assert ptr[0] == 0 and ptr[-1] == sp.size and (np.diff(ptr) >= 1).all()
    for e in range(len(g.ep_pin)):
        row = sp[ptr[e]:ptr[e + 1]]
        assert (np.diff(row) > 0).all()
        assert set(row.tolist()) <= srcs
        assert (rat[ptr[e]:ptr[e + 1]] >= g.ep_rat[e] + 1.99).all()
