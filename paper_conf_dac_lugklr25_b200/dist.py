"""Scenario sharding across GPUs: one process per GPU.

A single graph does not shard (serial level dependency), so the
multi-GPU path is independent scenarios: rank r evaluates a contiguous block of
the scenario list on its own replica of the graph, OCV scenarios with the TNS
gradient and sizing candidates forward-only.  The only exchange happens once,
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


def evaluate_sharded(evaluate, scenarios, n_grad: int, num_arcs: int, rank: int, world: int, device, dist=None):
    """Evaluate `scenarios` sharded over `world` ranks.

    evaluate(list_of_scenarios, want_grad) -> (summaries [k, 3] float64 tensor, grad [E, 2] float32 or None)
    Scenarios with index < n_grad contribute to the gradient sum.  Returns
    (summaries [n, 3] float64 on `device`, grad_sum [num_arcs, 2] float32 on
    `device`), identical on every rank."""
    import torch
    n = len(scenarios)
    lo, hi, per = scenario_block(n, rank, world)
    mine = list(range(lo, hi))
    g_idx = [s for s in mine if s < n_grad]
    f_idx = [s for s in mine if s >= n_grad]
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
        summ[len(g_idx): len(g_idx) + len(f_idx)] = s_f
    if world > 1:
        parts = [torch.empty_like(summ) for _ in range(world)]
        dist.all_gather(parts, summ)
        allsum = torch.cat(parts)
        work.wait()
        summ = allsum[:n]
    else:
        summ = summ[:n]
    return summ, grad
