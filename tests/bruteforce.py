"""Brute-force references that pin the oracle (tests only).

Independent of oracle/oracle.c: timing paths are enumerated explicitly
(recursively over fanin arcs, with the unateness rule of Alg 1 l.8), and
each path's distribution is the sum of its arc means and variances (Eq 1-2,
P:L77-79) with corner mean + N_sigma * std (Eq 3).
"""
from __future__ import annotations

import types

import numpy as np

POS, NEG, NON = 0, 1, 2


def tiny_dag(seed, n_pins=8, p_edge=0.35, sigma0=False, dyadic=False, unate_p=(0.4, 0.45, 0.15),
             n_ep=None):
    """Random DAG on <= 9 pins in a shuffled caller order (graph object like synth.Graph)."""
    rng = np.random.default_rng(seed)
    n = n_pins
    topo = rng.permutation(n)        # topo[k] = caller id of the k-th pin in a hidden order
    arcs = []
    for a in range(n):
        for b in range(a + 1, n):
            if rng.random() < p_edge:
                arcs.append((topo[a], topo[b]))
                if rng.random() < 0.08:                      # occasional parallel arc
                    arcs.append((topo[a], topo[b]))
    if not arcs:
        arcs.append((topo[0], topo[1]))
    arcs = [arcs[i] for i in rng.permutation(len(arcs))]
    E = len(arcs)
    af = np.array([a for a, _ in arcs], np.int32)
    at = np.array([b for _, b in arcs], np.int32)
    un = rng.choice([POS, NEG, NON], size=E, p=unate_p).astype(np.uint8)
    mean = rng.uniform(1.0, 20.0, (E, 2))
    sig = np.zeros((E, 2)) if sigma0 else rng.uniform(0.0, 3.0, (E, 2))
    smean = rng.uniform(0.0, 10.0, (n, 2))
    ssig = np.zeros((n, 2)) if sigma0 else rng.uniform(0.0, 2.0, (n, 2))
    if dyadic:
        mean = np.round(mean * 64) / 64
        smean = np.round(smean * 64) / 64
    has_out = np.zeros(n, bool)
    has_out[af] = True
    sinks = np.nonzero(~has_out)[0]
    if n_ep is None:
        eps = sinks
    else:
        eps = rng.choice(n, size=min(n_ep, n), replace=False)
    rat = rng.uniform(10.0, 60.0, (len(eps), 2))
    if dyadic:
        rat = np.round(rat * 64) / 64
    return types.SimpleNamespace(
        num_pins=n, arc_from=af, arc_to=at, arc_unate=un,
        arc_class=np.zeros(E, np.uint8),
        arc_mean=mean.astype(np.float32).astype(np.float64) if not dyadic else mean,
        arc_sigma=sig.astype(np.float32).astype(np.float64),
        src_mean=smean, src_sigma=ssig,
        ep_pin=np.asarray(eps, np.int32), ep_rat=rat, meta={})


def layered_equal_variance(seed, widths=(3, 3, 2, 2), s0=1.5, sa=2.0):
    """Strictly layered DAG (every arc joins consecutive layers), one sigma s0 on every source and
    one sigma sa on every arc and rf: every path into a layer-l pin carries variance s0^2 + l*sa^2."""
    rng = np.random.default_rng(seed)
    layers, n = [], 0
    for w in widths:
        layers.append(list(range(n, n + w)))
        n += w
    arcs = []
    for l in range(1, len(layers)):
        for b in layers[l]:
            srcs = [a for a in layers[l - 1] if rng.random() < 0.7] or [layers[l - 1][0]]
            arcs += [(a, b) for a in srcs]
    E = len(arcs)
    lvl = np.zeros(n, int)
    for l, ps in enumerate(layers):
        lvl[ps] = l
    g = types.SimpleNamespace(
        num_pins=n, arc_class=np.zeros(E, np.uint8), arc_from=np.array([a for a, _ in arcs], np.int32),
        arc_to=np.array([b for _, b in arcs], np.int32),
        arc_unate=rng.choice(3, size=E, p=[0.4, 0.4, 0.2]).astype(np.uint8),
        arc_mean=rng.uniform(1.0, 9.0, size=(E, 2)).astype(np.float32).astype(np.float64), arc_sigma=np.full((E, 2), sa),
        src_mean=np.where(lvl[:, None] == 0, rng.uniform(0.0, 3.0, size=(n, 2)), 0.0).astype(np.float32).astype(np.float64),
        src_sigma=np.where(lvl[:, None] == 0, np.full((n, 2), s0), 0.0),
        ep_pin=np.array(layers[-1], np.int32), ep_rat=np.full((len(layers[-1]), 2), 25.0))
    return g, lvl


def source_transitions(rf, u):
    if u == POS:
        return [rf]
    if u == NEG:
        return [1 - rf]
    return [rf, 1 - rf]


def enumerate_paths(g):
    """paths[(pin, rf)] = list of (mean_sum, var_sum, frozenset of (arc, rf) hops)."""
    n = g.num_pins
    fanin = [[] for _ in range(n)]
    for e in range(len(g.arc_from)):
        fanin[int(g.arc_to[e])].append(e)
    memo = {}

    def rec(i, rf):
        key = (i, rf)
        if key in memo:
            return memo[key]
        if not fanin[i]:
            out = [(float(g.src_mean[i][rf]), float(g.src_sigma[i][rf]) ** 2, ())]
        else:
            out = []
            for e in fanin[i]:
                j = int(g.arc_from[e])
                for s in source_transitions(rf, int(g.arc_unate[e])):
                    for m, v, hops in rec(j, s):
                        out.append((m + float(g.arc_mean[e][rf]), v + float(g.arc_sigma[e][rf]) ** 2,
                                    hops + ((e, rf),)))
        memo[key] = out
        return out

    return {(i, rf): rec(i, rf) for i in range(n) for rf in (0, 1)}


def corner(m, v, n_sigma):
    return m + n_sigma * np.sqrt(v)


def trace_critical(g, win_arc, win_s, pin, rf):
    """Follow the oracle's recorded winners back to a source: list of (arc, rf) hops."""
    hops = []
    i, r = pin, rf
    while win_arc[i][r] >= 0:
        e = int(win_arc[i][r])
        s = int(win_s[i][r])
        hops.append((e, r))
        i, r = int(g.arc_from[e]), s
    return i, r, hops
