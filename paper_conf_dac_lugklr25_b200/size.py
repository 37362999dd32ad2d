"""INSTA-Size without PrimeTime.

The paper's gradient-based gate sizer: a backward pass on TNS gives every
"stage" (a cell arc plus its driving net arc) a timing gradient; stages above a
threshold are taken most-critical first; for each, the library option with the
largest delay improvement on that stage is committed and rolled back if TNS
degrades; the 3-hop neighbourhood of a committed stage is blocked for the rest
of the iteration.  PrimeTime's estimate_eco (the delay estimate of a
library swap) is out of scope; a seeded synthetic library table stands in for
it (`library_options`).

Host orchestration only: every timing step runs in libinsta.so through the C
ABI -- insta_forward (incremental cone pass after insta_update_arcs),
insta_backward_update (the reverse-cone incremental backward), insta_stage_gradients,
insta_select_stages.
"""
from __future__ import annotations

import dataclasses

import numpy as np

from . import synth

# synthetic library: cell-arc delay factors of the alternative sizes of a cell;
# an upsized cell loads its input nets more (input-net factor 1 + 0.4 (1 - f))
LIB_FACTORS = (0.70, 0.80, 0.90, 1.10)


@dataclasses.dataclass
class SizeResult:
    tns0: float
    tns: float
    wns: float
    trials: int
    commits: int
    history: list          # (iteration, trial, tns after the trial, committed?)
    arc_mean: np.ndarray   # final annotation (caller order)
    arc_sigma: np.ndarray


class _Netlist:
    """Cell structure from the graph: cell arcs by output pin, input nets by pin, undirected adjacency."""

    def __init__(self, g):
        N = int(g.num_pins)
        af, at = np.asarray(g.arc_from), np.asarray(g.arc_to)
        cls = np.asarray(g.arc_class)
        self.cell = np.nonzero(cls == synth.CELL)[0]
        order = self.cell[np.argsort(at[self.cell], kind="stable")]
        self.cell_by_out = {}
        for a in order:
            self.cell_by_out.setdefault(int(at[a]), []).append(int(a))
        net = np.nonzero(cls == synth.NET)[0]
        self.net_into = {int(at[a]): int(a) for a in net}
        nbr = [[] for _ in range(N)]
        for a, b in zip(af.tolist(), at.tolist()):
            nbr[a].append(b)
            nbr[b].append(a)
        self.nbr = nbr

    def hops(self, pins, k):
        """Pins within k undirected arc hops of `pins`."""
        seen = set(pins)
        front = list(pins)
        for _ in range(k):
            nxt = []
            for p in front:
                for q in self.nbr[p]:
                    if q not in seen:
                        seen.add(q)
                        nxt.append(q)
            front = nxt
        return seen


def library_options(g, nl: _Netlist, out_pin: int, mean: np.ndarray, sigma: np.ndarray):
    """The estimate table of one cell: per library option, (arc ids, new mean, new sigma) of the cell's arcs
    and its input nets (mean and sigma scaled alike, fp32)."""
    arcs = nl.cell_by_out[out_pin]
    nets = [nl.net_into[int(g.arc_from[a])] for a in arcs if int(g.arc_from[a]) in nl.net_into]
    ids = np.array(arcs + nets, np.int32)
    opts = []
    for f in LIB_FACTORS:
        fac = np.array([f] * len(arcs) + [1.0 + 0.4 * (1.0 - f)] * len(nets))[:, None]
        opts.append((ids, (mean[ids] * fac).astype(np.float32), (sigma[ids] * fac).astype(np.float32)))
    return opts


def insta_size(G, g, iterations: int = 2, per_iter: int = 25, threshold: float = 0.0, n_sigma: float = 3.0,
               tau: float = 0.0, hops: int = 3, max_trials: int | None = None) -> SizeResult:
    """Run INSTA-Size on an insta.Graph `G` built from synth graph `g` (which must carry arc_class)."""
    nl = _Netlist(g)
    mean = np.asarray(g.arc_mean, np.float32).copy()
    sigma = np.asarray(g.arc_sigma, np.float32).copy()
    s = G.forward(n_sigma, tau)
    tns0 = tns = s.tns
    history, trials, commits = [], 0, 0
    d = G._torch.zeros((g.num_arcs, 2), dtype=G._torch.float32, device=G.device)
    for it in range(iterations):
        # the TNS gradient, kept current by the reverse-cone backward after the previous
        # iteration's cone passes (insta_backward_update; bit-identical to insta_backward)
        G.backward_update(d)
        sg = G.stage_gradients(d)
        order = G.select_stages(sg, threshold).cpu().numpy()
        blocked = set()
        done = 0
        for arc in order.tolist():
            if done >= per_iter or (max_trials is not None and trials >= max_trials):
                break
            out_pin = int(g.arc_to[arc])
            in_pin = int(g.arc_from[arc])
            if out_pin in blocked or in_pin in blocked:
                continue
            # the option with the largest delay improvement on this stage (cell arc + driving net arc)
            stage = [arc] + ([nl.net_into[in_pin]] if in_pin in nl.net_into else [])
            best, best_gain = None, 0.0
            for ids, nm, ns_ in library_options(g, nl, out_pin, mean, sigma):
                pos = {int(a): k for k, a in enumerate(ids)}
                gain = float(sum(nm[pos[a]].sum() - mean[a].sum() for a in stage if a in pos))
                if gain < best_gain:
                    best, best_gain = (ids, nm, ns_), gain
            if best is None:
                continue
            ids, nm, ns_ = best
            old_m, old_s = mean[ids].copy(), sigma[ids].copy()
            G.update_arcs(ids, nm, ns_, incremental=True)
            s = G.forward(n_sigma, tau)
            trials += 1
            ok = s.tns > tns
            if ok:                       # commit
                tns = s.tns
                mean[ids], sigma[ids] = nm, ns_
                commits += 1
                done += 1
                blocked |= nl.hops([out_pin, in_pin], hops)
            else:                        # roll back (TNS degraded or unchanged)
                G.update_arcs(ids, old_m, old_s, incremental=True)
                G.forward(n_sigma, tau)
            history.append((it, trials, float(s.tns), bool(ok)))
    s = G.forward(n_sigma, tau)
    return SizeResult(tns0=float(tns0), tns=float(s.tns), wns=float(s.wns), trials=trials, commits=commits,
                      history=history, arc_mean=mean, arc_sigma=sigma)
