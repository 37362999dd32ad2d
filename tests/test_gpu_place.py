"""GPU parity of the Eq 7 timing objective vs the oracle.

Loss within 1e-9 relative (fp64 sums of fp32 inputs on both sides, different
order); gradients are sums of +-lambda*w_k (fp64, rounded to fp32 once): within
1e-6 relative of the oracle's; Eq 8's norm ratio against numpy.linalg.norm.
The weights come from the GPU's own TNS backward, as in INSTA-Place.
"""
import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_timing_loss_parity(cfg):
    import torch
    g = synth.generate(cfg)
    rng = np.random.default_rng(11)
    x = rng.uniform(0, 1000, g.num_pins).astype(np.float32)
    y = rng.uniform(0, 1000, g.num_pins).astype(np.float32)
    G = insta.Graph(g)
    G.forward(3.0, 0.0)
    d = G.backward()
    w = -(d[:, 0] + d[:, 1])                       # R21: arc sensitivity >= 0
    L, gx, gy = G.timing_loss(x, y, w, lambda_rc=1e-3)
    Lg, gx, gy, w = float(L.item()), gx.cpu().numpy(), gy.cpu().numpy(), w.cpu().numpy()
    G.close()
    assert (w >= 0).all() and (w > 0).any()
    Lo, ox, oy = oracle.timing_loss(g, x, y, w, float(np.float32(1e-3)))   # the ABI takes lambda as float
    assert Lg == pytest.approx(Lo, rel=1e-9)
    assert np.allclose(gx, ox, rtol=1e-6, atol=1e-9)
    assert np.allclose(gy, oy, rtol=1e-6, atol=1e-9)
    a = torch.as_tensor(rng.normal(size=2 * g.num_pins).astype(np.float32), device="cuda")   # as long as b
    b = torch.as_tensor(np.concatenate([gx, gy]), device="cuda")
    r = float(insta.grad_norm_ratio(a, b).item())
    assert r == pytest.approx(np.linalg.norm(a.cpu().numpy().astype(np.float64)) /
                              np.linalg.norm(np.concatenate([gx, gy]).astype(np.float64)), rel=1e-9)


def test_timing_loss_heavy_fanout_and_determinism():
    """C2 has high-fanout nets (the warp-per-pin gradient path); two calls are bit-identical."""
    g = synth.generate("C2")
    rng = np.random.default_rng(5)
    x = rng.uniform(0, 1000, g.num_pins).astype(np.float32)
    y = rng.uniform(0, 1000, g.num_pins).astype(np.float32)
    w = rng.uniform(0, 1, g.num_arcs).astype(np.float32)
    G = insta.Graph(g)
    r1 = [t.cpu().numpy() for t in G.timing_loss(x, y, w, 0.5)]
    r2 = [t.cpu().numpy() for t in G.timing_loss(x, y, w, 0.5)]
    G.close()
    for a, b in zip(r1, r2):
        assert np.array_equal(a, b)
    Lo, ox, oy = oracle.timing_loss(g, x, y, w, 0.5)
    assert np.allclose(r1[1], ox, rtol=1e-6, atol=1e-6)
    fo = np.bincount(g.arc_from, minlength=g.num_pins)
    wide = fo > 32
    assert wide.any()
    assert np.allclose(r1[1][wide], ox[wide], rtol=1e-6, atol=1e-6)


def test_grad_norm_ratio_rejects_mismatched_lengths():
    import torch
    with pytest.raises(ValueError):
        insta.grad_norm_ratio(torch.ones(10, device="cuda"), torch.ones(12, device="cuda"))
