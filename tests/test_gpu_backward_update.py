"""Incremental backward (P:L156 INSTA-Size): after cone
passes, insta_backward_update re-runs the Eq 6 chain only in the reverse cone of what
changed and must equal a full insta_backward on the same state bit for bit."""
import numpy as np
import pytest
import torch

import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth

pytestmark = pytest.mark.gpu

CONE = 10 ** 9   # cone_max: take the cone pass whatever the update size


def bits(t):
    return t.cpu().numpy().view(np.uint32)


@pytest.mark.parametrize("tau", [0.0, 1.0])
@pytest.mark.parametrize("cfg,frac", [("C1", 0.01), ("C2", 0.0002), ("C2", 1e-5)])
def test_update_equals_full_backward(cfg, frac, tau):
    g = synth.generate(cfg)
    G = insta.Graph(g)
    G.forward(3.0, tau)
    out = torch.zeros((g.num_arcs, 2), dtype=torch.float32, device="cuda")
    assert G.backward_update(out) is False           # first call: full backward + snapshot
    assert np.array_equal(bits(out), bits(G.backward()))
    reran = []
    for step in range(4):
        ids, m, s = synth.sizing_step(g, 40 + step, frac=frac)
        G.update_arcs(ids, m, s, incremental=True)
        G.forward(3.0, tau, cone_max=CONE)
        assert G.backward_update(out) is True
        reran.append(G.last_backward_stats())
        ref = G.backward()
        assert np.array_equal(bits(out), bits(ref)), (step, int((bits(out) != bits(ref)).sum()))
    assert max(reran) > 0
    # a full forward in between: the next update runs the full backward
    ids, m, s = synth.sizing_step(g, 99, frac=frac)
    G.update_arcs(ids, m, s, incremental=False)
    G.forward(3.0, tau)
    assert G.backward_update(out) is False
    assert np.array_equal(bits(out), bits(G.backward()))
    G.close()


def test_update_small_change_is_a_small_cone():
    g = synth.generate("C2")
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    out = torch.zeros((g.num_arcs, 2), dtype=torch.float32, device="cuda")
    G.backward_update(out)
    ids, m, s = synth.sizing_step(g, 7, frac=1e-5)
    G.update_arcs(ids, m, s, incremental=True)
    G.forward(3.0, 0.0)
    assert G.backward_update(out) is True
    n = G.last_backward_stats()
    assert n < G.schedule()["num_heads"] // 10, n
    assert np.array_equal(bits(out), bits(G.backward()))
    # unchanged state: nothing to re-run, result unchanged
    G.update_arcs(ids, m, s, incremental=True)
    G.forward(3.0, 0.0)
    assert G.backward_update(out) is True
    assert G.last_backward_stats() == 0
    assert np.array_equal(bits(out), bits(G.backward()))
    G.close()


def test_update_other_buffer_or_options_runs_full():
    g = synth.generate("C1")
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    a = torch.zeros((g.num_arcs, 2), dtype=torch.float32, device="cuda")
    b = torch.zeros_like(a)
    assert G.backward_update(a) is False
    assert G.backward_update(b) is False             # another buffer
    G.forward(2.5, 0.0)                              # other n_sigma (a full pass anyway)
    assert G.backward_update(b) is False
    assert np.array_equal(bits(b), bits(G.backward()))
    G.close()


def test_update_policy_many_arcs_runs_full():
    # more than max(64, E / 5e4) arcs re-annotated since the snapshot: the full backward (still exact)
    g = synth.generate("C2")
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    out = torch.zeros((g.num_arcs, 2), dtype=torch.float32, device="cuda")
    G.backward_update(out)
    ids, m, s = synth.sizing_step(g, 5, frac=0.002)
    assert len(ids) > 64
    G.update_arcs(ids, m, s, incremental=True)
    G.forward(3.0, 0.0, cone_max=CONE)
    assert G.backward_update(out) is False
    assert np.array_equal(bits(out), bits(G.backward()))
    G.close()


@pytest.mark.slow
def test_update_c4_one_cell_steps():
    """C4 (15M pins) at the headline scale: one-cell sizing steps through the cone pass, the kept
    TNS gradient brought up to date by the reverse cone equals a full backward bit for bit."""
    g = synth.generate("C4")
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    out = torch.zeros((g.num_arcs, 2), dtype=torch.float32, device="cuda")
    assert G.backward_update(out) is False
    for step in range(3):
        ids, m, s = synth.sizing_step(g, 60 + step, frac=1e-6)
        G.update_arcs(ids, m, s, incremental=True)
        G.forward(3.0, 0.0)
        assert G.backward_update(out) is True
        assert np.array_equal(bits(out), bits(G.backward())), step
    G.close()
