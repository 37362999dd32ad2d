"""Scenario sharding across GPUs: one process per GPU.

A single graph does not shard (serial level dependency), so the
multi-GPU path is independent scenarios: rank r evaluates, on its own replica
of the graph, a contiguous block of the gradient (OCV) scenarios and a
contiguous block of the forward-only (sizing-candidate) scenarios -- the two
classes are split separately, so every rank gets the same mix (an OCV scenario
with its backward costs ~15x a one-cell candidate on the cone pass; one block
of the whole list would put all OCV work on the first half of the ranks).  The only exchange happens once,
at the end: an all_gather of the per-scenario summaries {wns, tns, #viol} and
an all_reduce(SUM) of the gradient sum over scenarios.  With the nccl backend
these run over NVLink; the host logic is backend-agnostic (gloo tests).
"""
from __future__ import annotations


def scenario_block(n: int, rank: int, world: int):
    """Contiguous block [lo, hi) of n scenarios owned by `rank`."""
    per = (n + world - 1) // world
    lo = min(n, rank * per)
    return lo, min(n, lo + per), per


def evaluate_sharded(evaluate, scenarios, n_grad: int, num_arcs: int, rank: int, world: int, device, dist=None,
                     timing: dict | None = None):
    """Evaluate `scenarios` sharded over `world` ranks.

    evaluate(list_of_scenarios, want_grad) -> (summaries [k, 3] float64 tensor, grad [E, 2] float32 or None)
    Scenarios with index < n_grad contribute to the gradient sum.  Returns
    (summaries [n, 3] float64 on `device`, grad_sum [num_arcs, 2] float32 on
    `device`), identical on every rank.  timing (optional dict): 'collective_ms' = device time from the
    end of this rank's evaluations to the gathered result (the all_gather plus what is left of the
    overlapped all_reduce; CUDA events on the current stream)."""
    import torch
    n = len(scenarios)
    n_f = n - n_grad
    glo, ghi, gper = scenario_block(n_grad, rank, world)
    flo, fhi, fper = scenario_block(n_f, rank, world)
    g_idx = list(range(glo, ghi))
    f_idx = [n_grad + s for s in range(flo, fhi)]
    per = gper + fper
    summ = torch.zeros((per, 3), dtype=torch.float64, device=device)
    grad = torch.zeros((num_arcs, 2), dtype=torch.float32, device=device)
    if g_idx:
        s_g, d_g = evaluate([scenarios[s] for s in g_idx], True)
        summ[: len(g_idx)] = s_g
        grad += d_g
    # the gradient sum is final once the gradient scenarios are done: its
    # all_reduce runs (on NCCL's stream) while the forward-only scenarios compute
    work = dist.all_reduce(grad, op=dist.ReduceOp.SUM, async_op=True) if world > 1 else None
    if f_idx:
        s_f, _ = evaluate([scenarios[s] for s in f_idx], False)
        summ[gper: gper + len(f_idx)] = s_f
    ev0 = ev1 = None
    if timing is not None and world > 1 and torch.cuda.is_available() and str(device).startswith("cuda"):
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record()
    if world > 1:
        parts = [torch.empty_like(summ) for _ in range(world)]
        dist.all_gather(parts, summ)
        out = torch.empty((n, 3), dtype=torch.float64, device=device)
        for r, part in enumerate(parts):   # back to scenario order
            a, b, _ = scenario_block(n_grad, r, world)
            c, d, _ = scenario_block(n_f, r, world)
            out[a:b] = part[: b - a]
            out[n_grad + c: n_grad + d] = part[gper: gper + d - c]
        work.wait()
        summ = out
        if ev0 is not None:
            ev1.record()
            ev1.synchronize()
            timing["collective_ms"] = ev0.elapsed_time(ev1)
    else:
        summ = torch.cat([summ[: len(g_idx)], summ[gper: gper + len(f_idx)]])
    return summ, grad
