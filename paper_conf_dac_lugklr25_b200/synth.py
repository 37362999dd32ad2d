"""Seeded synthetic timing-graph generator (input recipe only).

This module is the ONE piece shared by the CUDA path's tests/bench and the CPU
oracle's tests.  It draws netlist-shaped timing DAGs and their arc/SP/EP values;
it holds none of the method's arithmetic (no propagation, no merge, no slack).
Everything it returns is plain numpy, in CALLER order (shuffled ids), in the
layout of `insta_graph_desc` (include/insta.h).

Recipe.  The paper gives only cell
and pin counts for its designs (block-1 4M cells / 15M pins,
i.e. ~3.75 pins per cell), so the structure below is a stated assumption:

* logic cells with k in {1,2,3,4} inputs (p = .10/.30/.35/.25, mean 2.75), one
  output each; flops contribute a startpoint pin (Q, indeg 0) and an endpoint
  pin (D); clock pins are not propagated (clock arrival is an SP attribute,
  PAPER.md L62).
* each cell gets a stage depth d in 1..D with P(d) ~ (D+1-d); a spine chain
  guarantees depth D, so pin levels ~ 2D+1.
* a cell input at depth d is driven by a net arc from depth d-1 with
  probability 0.7, else from a uniform shallower depth (0 = flop Q).
* drivers carry power-law fanout weights P(f) ~ f^-alpha on [1, cap]; sinks are
  assigned first to cover every driver once, then in proportion to weight.
  C2/C4 add ~10 high-fanout nets (10^3 .. 2*10^4 sinks).
* cell arcs: NEG .55 / POS .40 / NON .05; net arcs POS (PAPER.md L62, L70 l.8).
* endpoint D pins are driven from depths >= D/2; dangling cell outputs are POs
  and become endpoints too.
* values (ps): cell mu_R ~ LogNormal(ln 12, .45), mu_F = mu_R*U(.8,1.25);
  net mu_R ~ LogNormal(ln 2, .8), mu_F = mu_R*U(.9,1.1); sigma = mu*U(.02,.08)
  (cell) or mu*U(0,.05) (net); SP mu ~ N(150,15) clipped >= 0, sigma ~ U(1,4);
  RAT = T_clk + N(150,15) - U(5,15) per rf.
* dyadic mode: every mu and RAT on a 2^-6 ps grid, every sigma = 0 -- fp32 sums
  are then exact, so GPU and oracle must agree bit for bit.
"""
from __future__ import annotations

import dataclasses
import numpy as np

POS, NEG, NON = 0, 1, 2
NET, CELL = 0, 1


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    pins: int            # target pin count
    depth: int           # stage depth D (pin levels ~ 2D+1)
    ep_frac: float       # target endpoint fraction
    cap: int             # fanout weight cap
    alpha: float         # power-law exponent of fanout weights
    n_hf: int            # high-fanout nets
    hf_lo: int
    hf_hi: int
    seed: int
    t_clk: float         # clock period (ps); see tools/calibrate_tclk.py


# T_clk values were written by tools/calibrate_tclk.py (which calls only the
# oracle): the 85th percentile of hard-mode EP arrival minus the RAT offset, so
# that ~10-20% of endpoints violate in hard mode.
CONFIGS = {
    "C1": Config("C1", 2_000, 15, 0.10, 16, 1.66, 0, 0, 0, 101, 320.0),
    "C2": Config("C2", 200_000, 50, 0.05, 2_000, 2.25, 10, 1_000, 20_000, 202, 1165.0),
    "C3": Config("C3", 2_000_000, 60, 0.03, 4_000, 2.26, 10, 1_000, 20_000, 303, 1446.0),
    "C4": Config("C4", 15_000_000, 80, 0.027, 4_000, 2.26, 10, 1_000, 20_000, 404, 1977.0),
}
CONFIGS["C5"] = dataclasses.replace(CONFIGS["C4"], name="C5", seed=505)


@dataclasses.dataclass
class Graph:
    """A timing graph in caller order (the layout of insta_graph_desc)."""
    num_pins: int
    arc_from: np.ndarray   # int32 [E]
    arc_to: np.ndarray     # int32 [E]
    arc_unate: np.ndarray  # uint8 [E]  POS/NEG/NON
    arc_class: np.ndarray  # uint8 [E]  NET/CELL
    arc_mean: np.ndarray   # float32 [E,2] {R,F} of the sink transition
    arc_sigma: np.ndarray  # float32 [E,2]
    src_mean: np.ndarray   # float32 [N,2] (read only at indeg-0 pins)
    src_sigma: np.ndarray  # float32 [N,2]
    ep_pin: np.ndarray     # int32 [P]
    ep_rat: np.ndarray     # float32 [P,2]
    meta: dict

    @property
    def num_arcs(self) -> int:
        return int(self.arc_from.shape[0])

    @property
    def num_endpoints(self) -> int:
        return int(self.ep_pin.shape[0])


def _powerlaw(rng, n, alpha, cap):
    """Continuous power law on [1, cap+1), floored: P(f) ~ f^-alpha."""
    u = rng.random(n)
    a1 = 1.0 - alpha
    hi = (cap + 1.0) ** a1
    f = (1.0 + u * (hi - 1.0)) ** (1.0 / a1)
    return np.floor(f)


def generate(cfg: Config | str, dyadic: bool = False, pins: int | None = None) -> Graph:
    """Draw the graph of config `cfg` (name or Config).  `pins` overrides the size."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    if pins is not None:
        cfg = dataclasses.replace(cfg, pins=int(pins))
    rng = np.random.default_rng(cfg.seed)
    D = cfg.depth
    N_t = cfg.pins

    # ---- counts -----------------------------------------------------------
    F = max(2, int(round(cfg.ep_frac * N_t * 0.9)))          # flops
    C = max(D, int(round((N_t - 2 * F) / 3.75)))            # logic cells
    k = rng.choice(np.array([1, 2, 3, 4]), size=C, p=[0.10, 0.30, 0.35, 0.25]).astype(np.int64)
    # stage depth, front-loaded; the first D cells are the spine (depth 1..D)
    pd = (D + 1 - np.arange(1, D + 1)).astype(np.float64)
    depth = rng.choice(np.arange(1, D + 1), size=C, p=pd / pd.sum()).astype(np.int64)
    depth[:D] = np.arange(1, D + 1)
    if D >= 1:
        k[:D] = np.maximum(k[:D], 1)

    # ---- pin numbering (internal, shuffled at the end) ---------------------
    # [0,F) flop Q (SP) ; [F,2F) flop D (EP) ; then per cell: k inputs then output
    n_in = int(k.sum())
    in_base = 2 * F
    cell_in_start = in_base + np.concatenate([[0], np.cumsum(k)[:-1]])   # first input pin of cell
    out_base = in_base + n_in
    cell_out = out_base + np.arange(C)
    N = out_base + C

    # ---- drivers: SP pins (depth 0) and cell outputs (depth d) -------------
    drv_pin = np.concatenate([np.arange(F), cell_out])
    drv_depth = np.concatenate([np.zeros(F, np.int64), depth])
    drv_w = _powerlaw(rng, drv_pin.shape[0], cfg.alpha, cfg.cap)

    # ---- sinks: cell input pins, and flop D pins ---------------------------
    sink_pin = np.concatenate([in_base + np.arange(n_in), F + np.arange(F)])
    cell_of_in = np.repeat(np.arange(C), k)
    d_in = depth[cell_of_in]
    r = rng.random(n_in)
    shallower = np.floor(rng.random(n_in) * np.maximum(d_in - 1, 1)).astype(np.int64)
    tgt_in = np.where((r < 0.7) | (d_in <= 1), d_in - 1, shallower)
    tgt_ep = rng.integers(D // 2, D + 1, size=F)
    sink_tgt = np.concatenate([tgt_in, tgt_ep])
    # spine: input 0 of spine cell at depth d is driven by spine cell at depth d-1
    spine_in = cell_in_start[:D]
    sink_tgt[spine_in - in_base] = np.arange(0, D)

    sink_drv = np.empty(sink_pin.shape[0], np.int64)   # driver pin per sink
    order_d = np.argsort(drv_depth, kind="stable")
    dd_sorted = drv_depth[order_d]
    dptr = np.searchsorted(dd_sorted, np.arange(D + 2))
    order_s = np.argsort(sink_tgt, kind="stable")
    st_sorted = sink_tgt[order_s]
    sptr = np.searchsorted(st_sorted, np.arange(D + 2))
    for d in range(D + 1):
        drv = order_d[dptr[d]:dptr[d + 1]]
        snk = order_s[sptr[d]:sptr[d + 1]]
        if snk.size == 0:
            continue
        if drv.size == 0:  # cannot happen for d <= D-? but keep safe: fall back to SPs
            drv = order_d[dptr[0]:dptr[1]]
        snk = rng.permutation(snk)
        ncov = min(snk.size, drv.size)
        cov = rng.permutation(drv)[:ncov]
        sink_drv[snk[:ncov]] = drv_pin[cov]
        rest = snk[ncov:]
        if rest.size:
            cw = np.cumsum(drv_w[drv])
            pick = np.searchsorted(cw, rng.random(rest.size) * cw[-1], side="right")
            pick = np.minimum(pick, drv.size - 1)
            sink_drv[rest] = drv_pin[drv[pick]]
    # spine edges fixed after the random assignment
    for d in range(1, D + 1):
        sp_sink = spine_in[d - 1] - in_base
        sink_drv[sp_sink] = (np.int64(0) if d == 1 else cell_out[d - 2])

    # ---- high-fanout nets ----------------------------------------------------
    if cfg.n_hf > 0:
        shallow = np.nonzero(depth[D:] <= max(1, D // 2))[0] + D
        hf_cells = rng.choice(shallow, size=min(cfg.n_hf, shallow.size), replace=False)
        budget = int(0.03 * sink_pin.shape[0])     # high-fanout sinks <= 3% of all sinks
        for c in hf_cells:
            size = int(np.exp(rng.uniform(np.log(cfg.hf_lo), np.log(cfg.hf_hi))))
            size = min(size, budget)
            budget -= size
            if size < cfg.hf_lo // 2:
                break
            ok = np.nonzero(d_in > depth[c])[0]
            ok = ok[~np.isin(ok, spine_in - in_base)]
            if ok.size == 0:
                continue
            chosen = rng.choice(ok, size=min(size, ok.size), replace=False)
            sink_drv[chosen] = cell_out[c]

    # ---- arcs -----------------------------------------------------------------
    net_from = sink_drv
    net_to = sink_pin
    cell_from = in_base + np.arange(n_in)
    cell_to = cell_out[cell_of_in]
    E_net, E_cell = net_from.shape[0], cell_from.shape[0]
    a_from = np.concatenate([net_from, cell_from])
    a_to = np.concatenate([net_to, cell_to])
    a_class = np.concatenate([np.full(E_net, NET, np.uint8), np.full(E_cell, CELL, np.uint8)])
    u = rng.random(E_cell)
    cell_un = np.where(u < 0.55, NEG, np.where(u < 0.95, POS, NON)).astype(np.uint8)
    a_unate = np.concatenate([np.full(E_net, POS, np.uint8), cell_un])
    E = E_net + E_cell

    # ---- values (ps) ---------------------------------------------------------
    mean = np.empty((E, 2), np.float64)
    sig = np.empty((E, 2), np.float64)
    mu_r = rng.lognormal(np.log(2.0), 0.8, E_net)
    mean[:E_net, 0] = mu_r
    mean[:E_net, 1] = mu_r * rng.uniform(0.9, 1.1, E_net)
    sig[:E_net] = mean[:E_net] * rng.uniform(0.0, 0.05, (E_net, 2))
    mu_r = rng.lognormal(np.log(12.0), 0.45, E_cell)
    mean[E_net:, 0] = mu_r
    mean[E_net:, 1] = mu_r * rng.uniform(0.8, 1.25, E_cell)
    sig[E_net:] = mean[E_net:] * rng.uniform(0.02, 0.08, (E_cell, 2))

    src_mean = np.zeros((N, 2), np.float64)
    src_sig = np.zeros((N, 2), np.float64)
    src_mean[:F] = np.maximum(rng.normal(150.0, 15.0, (F, 2)), 0.0)
    src_sig[:F] = rng.uniform(1.0, 4.0, (F, 2))

    # ---- endpoints: flop D pins + dangling cell outputs (POs) -----------------
    has_fo = np.zeros(N, bool)
    has_fo[a_from] = True
    po = cell_out[~has_fo[cell_out]]
    ep = np.concatenate([F + np.arange(F), po])
    P = ep.shape[0]
    base = rng.normal(150.0, 15.0, P)
    rat = np.stack([cfg.t_clk + base - rng.uniform(5.0, 15.0, P),
                    cfg.t_clk + base - rng.uniform(5.0, 15.0, P)], axis=1)

    if dyadic:
        g = 64.0
        mean = np.round(mean * g) / g
        sig[:] = 0.0
        src_mean = np.round(src_mean * g) / g
        src_sig[:] = 0.0
        rat = np.round(rat * g) / g

    # ---- shuffle caller ids ---------------------------------------------------
    pin_perm = rng.permutation(N)            # internal pin -> caller pin id
    arc_perm = rng.permutation(E)            # caller arc id -> internal arc
    inv = np.empty(N, np.int64)
    inv[:] = pin_perm
    s_mean = np.zeros((N, 2), np.float32)
    s_sig = np.zeros((N, 2), np.float32)
    s_mean[pin_perm] = src_mean
    s_sig[pin_perm] = src_sig
    ep_order = rng.permutation(P)
    meta = dict(config=cfg.name, seed=cfg.seed, dyadic=bool(dyadic), depth=D, flops=F,
                cells=C, pins=int(N), arcs=int(E), endpoints=int(P), t_clk=cfg.t_clk,
                net_arcs=int(E_net), cell_arcs=int(E_cell))
    return Graph(
        num_pins=int(N),
        arc_from=inv[a_from][arc_perm].astype(np.int32),
        arc_to=inv[a_to][arc_perm].astype(np.int32),
        arc_unate=a_unate[arc_perm].copy(),
        arc_class=a_class[arc_perm].copy(),
        arc_mean=mean[arc_perm].astype(np.float32),
        arc_sigma=sig[arc_perm].astype(np.float32),
        src_mean=s_mean,
        src_sigma=s_sig,
        ep_pin=inv[ep][ep_order].astype(np.int32),
        ep_rat=rat[ep_order].astype(np.float32),
        meta=meta,
    )


# ---------------------------------------------------------------------------
# Update streams (C3) and scenario parameters (C5): inputs, not arithmetic of
# the method.  Values are materialized in fp32 here exactly as a caller would.
# ---------------------------------------------------------------------------
def _cell_groups(g: Graph):
    """Caller arc ids grouped by sink pin for cell arcs (one group per cell)."""
    cell = np.nonzero(g.arc_class == CELL)[0]
    order = cell[np.argsort(g.arc_to[cell], kind="stable")]
    sinks = g.arc_to[order]
    starts = np.concatenate([[0], np.nonzero(np.diff(sinks))[0] + 1, [order.size]])
    return order, starts


def sizing_step(g: Graph, step: int, frac: float = 0.01, base_seed: int = 3030):
    """One gate-sizing style update (C3): returns (arc_ids int32, mean f32[n,2], sigma f32[n,2]).

    Picks random cells until ~`frac` of arcs are covered; scales the picked
    cell's arcs by U(.75,1.05) and its input net arcs by U(1.0,1.1) (mean and
    sigma alike)."""
    rng = np.random.default_rng(base_seed + step)
    order, starts = _cell_groups(g)
    ncell = starts.size - 1
    target = max(1, int(frac * g.num_arcs))
    # net arcs into each cell input pin, cell arcs into each cell output
    net = np.nonzero(g.arc_class == NET)[0]
    net_by_to = np.full(g.num_pins, -1, np.int64)
    net_by_to[g.arc_to[net]] = net
    scale = {}
    picked = rng.permutation(ncell)
    covered = 0
    for c in picked:
        arcs = order[starts[c]:starts[c + 1]]
        f = rng.uniform(0.75, 1.05)
        for a in arcs:
            scale[int(a)] = scale.get(int(a), 1.0) * f
        ins = g.arc_from[arcs]
        nets = net_by_to[ins]
        nets = nets[nets >= 0]
        for a in nets:
            scale[int(a)] = scale.get(int(a), 1.0) * rng.uniform(1.0, 1.1)
        covered = len(scale)
        if covered >= target:
            break
    ids = np.array(sorted(scale), np.int32)
    fac = np.array([scale[int(i)] for i in ids], np.float64)[:, None]
    return ids, (g.arc_mean[ids] * fac).astype(np.float32), (g.arc_sigma[ids] * fac).astype(np.float32)


def sizing_scenario(g: Graph, s: int, seed: int = 505, _cache={}):
    """Sizing-candidate scenario s (C5 scenarios 512..1023): one random cell's arcs
    scaled by U(.75, 1.05) and its input net arcs by U(1.0, 1.1) (mean and sigma
    alike), as a scenario dict for insta_forward_batch (fp32 override values)."""
    key = id(g)
    if key not in _cache:
        order, starts = _cell_groups(g)
        net = np.nonzero(g.arc_class == NET)[0]
        net_by_to = np.full(g.num_pins, -1, np.int64)
        net_by_to[g.arc_to[net]] = net
        _cache.clear()
        _cache[key] = (order, starts, net_by_to)
    order, starts, net_by_to = _cache[key]
    rng = np.random.default_rng([seed, s])
    c = int(rng.integers(starts.size - 1))
    arcs = order[starts[c]:starts[c + 1]]
    nets = net_by_to[g.arc_from[arcs]]
    nets = nets[nets >= 0]
    ids = np.concatenate([arcs, nets]).astype(np.int32)
    fac = np.concatenate([np.full(arcs.size, rng.uniform(0.75, 1.05)), rng.uniform(1.0, 1.1, nets.size)])[:, None]
    ids, first = np.unique(ids, return_index=True)
    fac = fac[first]
    return dict(n_sigma=3.0, derate_cell=1.0, derate_net=1.0, delta_arc=ids,
                delta_mean=(g.arc_mean[ids] * fac).astype(np.float32),
                delta_sigma=(g.arc_sigma[ids] * fac).astype(np.float32))


def c5_scenarios(g: Graph, n: int = 1024, n_ocv: int = 512, seed: int = 505):
    """The C5 workload: scenarios 0..n_ocv-1 are OCV (N_sigma, derates), the rest sizing candidates."""
    out = []
    for s in range(n):
        if s < n_ocv:
            ns, dc, dn = ocv_scenario(s, seed)
            out.append(dict(n_sigma=ns, derate_cell=dc, derate_net=dn))
        else:
            out.append(sizing_scenario(g, s, seed))
    return out


def ocv_scenario(s: int, seed: int = 505):
    """OCV scenario s (C5 scenarios 0..511): (n_sigma, derate_cell, derate_net)."""
    rng = np.random.default_rng([seed, s])
    return float(rng.uniform(2.5, 3.5)), float(rng.uniform(0.95, 1.10)), float(rng.uniform(0.95, 1.10))


# ---------------------------------------------------------------------------
# CPPR required-time table ("SP/EP attributes (e.g.
# clock arrival times, minimum required times)", P:L119 endpoint required times
# "associated with respective startpoints").  Structural input, no arithmetic
# of the method: for each endpoint, `per_ep` random backward walks over fanin
# arcs reach startpoints of its cone; each distinct one gets a clock-
# reconvergence credit U(2, 25) ps added to the endpoint's default required
# time (the common clock path removes pessimism, so RAT(ep, sp) >= RAT(ep)).
# ---------------------------------------------------------------------------
def cppr_rat_table(g, per_ep: int = 8, seed: int = 4242, dyadic: bool = False):
    """Returns (ptr int32[P+1], sp int32[M] caller pin ids ascending per endpoint, rat float32[M,2])."""
    rng = np.random.default_rng(seed)
    N, P = int(g.num_pins), int(np.asarray(g.ep_pin).shape[0])
    to = np.asarray(g.arc_to, np.int64)
    order = np.argsort(to, kind="stable")
    ptr = np.zeros(N + 1, np.int64)
    np.add.at(ptr, to + 1, 1)
    ptr = np.cumsum(ptr)
    src_of = np.asarray(g.arc_from, np.int64)[order]
    cur = np.repeat(np.asarray(g.ep_pin, np.int64), per_ep)
    while True:
        deg = ptr[cur + 1] - ptr[cur]
        live = deg > 0
        if not live.any():
            break
        pick = ptr[cur[live]] + (rng.random(int(live.sum())) * deg[live]).astype(np.int64)
        cur[live] = src_of[pick]
    pairs = np.unique(np.stack([np.repeat(np.arange(P), per_ep), cur], 1), axis=0)   # sorted (ep, sp)
    cnt = np.bincount(pairs[:, 0], minlength=P)
    rptr = np.concatenate([[0], np.cumsum(cnt)]).astype(np.int32)
    credit = rng.uniform(2.0, 25.0, pairs.shape[0])
    if dyadic:
        credit = np.round(credit * 64) / 64
    rat = np.asarray(g.ep_rat, np.float64).reshape(P, 2)[pairs[:, 0]] + credit[:, None]
    return rptr, pairs[:, 1].astype(np.int32), rat.astype(np.float32)
