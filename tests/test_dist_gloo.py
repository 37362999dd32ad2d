"""Multi-process scenario sharding with the gloo backend on CPU.

The sharded driver (paper_conf_dac_lugklr25_b200.dist) is run with world_size 2
using an oracle-backed evaluator (test stand-in for the GPU batch kernel); the
gathered per-scenario summaries and the reduced gradient sum must equal the
unsharded result."""
import os
import types

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_dac_lugklr25_b200 import dist as idist
from paper_conf_dac_lugklr25_b200 import synth


def materialize(g, sc):
    d = np.where(g.arc_class == synth.CELL, np.float32(sc["derate_cell"]), np.float32(sc["derate_net"]))
    d = d.astype(np.float32)[:, None]
    m = (g.arc_mean * d).astype(np.float32)
    s = (g.arc_sigma * d).astype(np.float32)
    if sc.get("delta_arc") is not None:
        m[sc["delta_arc"]] = sc["delta_mean"]
        s[sc["delta_arc"]] = sc["delta_sigma"]
    h = types.SimpleNamespace(**vars(g))
    h.arc_mean, h.arc_sigma = m, s
    return h


def oracle_eval(g):
    def ev(scs, want_grad):
        summ = np.zeros((len(scs), 3))
        grad = np.zeros((g.num_arcs, 2))
        for k, sc in enumerate(scs):
            h = materialize(g, sc)
            f = oracle.forward(h, sc["n_sigma"], 0.0)
            o = oracle.slack(h, f["A"])
            summ[k] = (o["wns"], o["tns"], o["num_viol"])
            if want_grad:
                grad += oracle.backward(h, sc["n_sigma"], 0.0)["d_mean"]
        return torch.from_numpy(summ), (torch.from_numpy(grad.astype(np.float32)) if want_grad else None)
    return ev


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = synth.generate("C1")
    scs = synth.c5_scenarios(g, n=11, n_ocv=5)
    summ, grad = idist.evaluate_sharded(oracle_eval(g), scs, 5, g.num_arcs, rank, world, "cpu", dist)
    if rank == 0:
        np.save(out + "_summ.npy", summ.numpy())
        np.save(out + "_grad.npy", grad.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_scenario_blocks_cover_exactly_once():
    for n in (1, 7, 1024, 1023):
        for w in (1, 2, 3, 8):
            seen = []
            for r in range(w):
                lo, hi, per = idist.scenario_block(n, r, w)
                assert hi - lo <= per
                seen += list(range(lo, hi))
            assert seen == list(range(n))


def test_sharded_equals_unsharded(tmp_path):
    g = synth.generate("C1")
    scs = synth.c5_scenarios(g, n=11, n_ocv=5)   # 5 OCV + 6 sizing: uneven blocks in both classes
    ref_summ, ref_grad = idist.evaluate_sharded(oracle_eval(g), scs, 5, g.num_arcs, 0, 1, "cpu")
    out = str(tmp_path / "r")
    port = 29500 + (os.getpid() % 1000)
    mp.spawn(_worker, args=(2, port, out), nprocs=2, join=True)
    summ = np.load(out + "_summ.npy")
    grad = np.load(out + "_grad.npy")
    assert np.array_equal(summ, ref_summ.numpy())
    assert np.allclose(grad, ref_grad.numpy(), rtol=1e-6, atol=1e-6)
    # OCV scenarios carry gradients, sizing candidates do not: the sum must be nonzero
    assert np.abs(grad).sum() > 0


def test_each_rank_gets_both_classes():
    # 1024 scenarios, 512 OCV: every rank of 2/4/8 evaluates 512/N of each class
    for w in (2, 4, 8):
        for r in range(w):
            a, b, _ = idist.scenario_block(512, r, w)
            c, d, _ = idist.scenario_block(512, r, w)
            assert b - a == 512 // w and d - c == 512 // w
