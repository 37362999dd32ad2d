"""Edge cases of the SURVEY §8(f) rows on the GPU: graphs without arcs, without endpoints, endpoints that
are startpoints, a wide-fanout driver, K larger than the number of startpoints."""
import types

import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta

pytestmark = pytest.mark.gpu


def _g(n, af, at, eps, unate=None, cls=None, seed=0):
    rng = np.random.default_rng(seed)
    E = len(af)
    return types.SimpleNamespace(
        num_pins=n, arc_from=np.asarray(af, np.int32), arc_to=np.asarray(at, np.int32),
        arc_unate=np.asarray(unate if unate is not None else [0] * E, np.uint8),
        arc_class=np.asarray(cls if cls is not None else [1] * E, np.uint8),
        arc_mean=rng.uniform(1, 10, (E, 2)).astype(np.float32), arc_sigma=rng.uniform(0.1, 1, (E, 2)).astype(np.float32),
        src_mean=rng.uniform(0, 5, (n, 2)).astype(np.float32), src_sigma=rng.uniform(0.1, 1, (n, 2)).astype(np.float32),
        ep_pin=np.asarray(eps, np.int32), ep_rat=np.full((len(eps), 2), 3.0, np.float32))


def test_no_arcs_endpoint_is_startpoint():
    g = _g(3, [], [], [1])
    G = insta.Graph(g)
    G.topk_forward(4, 3.0)
    s, sl, sp = G.topk_slack()
    q = G.topk_queues()
    assert int(sp.cpu()[0]) == 1 and int(q["sp"].cpu()[1, 0, 0]) == 1 and int(q["sp"].cpu()[1, 0, 1]) == -1
    c = G.clark_forward(3.0)
    assert c.tns == pytest.approx(s.tns, rel=1e-6)
    assert G.clark_backward().numel() == 0
    L, gx, gy = G.timing_loss(np.zeros(3), np.zeros(3), np.zeros(0))
    assert float(L.item()) == 0.0 and (gx.cpu() == 0).all()
    G.forward(3.0, 0.0)
    d = G.backward()
    assert G.select_stages(G.stage_gradients(d)).numel() == 0
    G.close()


def test_no_endpoints():
    g = _g(4, [0, 1, 2], [1, 2, 3], [])
    G = insta.Graph(g)
    G.topk_forward(2, 3.0)
    s, _, _ = G.topk_slack()
    assert s.tns == 0.0 and s.num_violations == 0
    c = G.clark_forward(3.0)
    assert c.tns == 0.0
    dm = G.clark_backward().cpu().numpy()
    assert (dm == 0).all()
    G.close()


def test_wide_driver_and_k_above_startpoints():
    # one driver with 100 sinks that reconverge in pairs; 3 startpoints, K = 8
    n_sink = 100
    af, at = [], []
    src = [0, 1, 2]
    drv = 3
    af += [0, 1, 2]
    at += [drv, drv, drv]
    for k in range(n_sink):
        af.append(drv)
        at.append(4 + k)
    out = 4 + n_sink
    for k in range(0, n_sink, 2):
        af += [4 + k, 4 + k + 1]
        at += [out + k // 2, out + k // 2]
    n = out + n_sink // 2
    eps = list(range(out, n))
    g = _g(n, af, at, eps, unate=[2] * len(af), seed=3)
    G = insta.Graph(g)
    G.topk_forward(8, 3.0)
    q = {k: v.cpu().numpy() for k, v in G.topk_queues().items()}
    oq = oracle.topk_forward(g, 3.0, 8)
    assert np.array_equal(q["sp"], oq["sp"])
    assert (q["sp"][eps][:, :, 3:] == -1).all()          # only 3 startpoints exist
    G.clark_forward(3.0)
    dm, ds = (x.cpu().numpy() for x in G.clark_backward(want_sigma=True))
    b = oracle.clark_backward(g, 3.0)
    assert np.allclose(dm, b["d_mean"], rtol=1e-3, atol=1e-3)
    rng = np.random.default_rng(0)
    x, y, w = rng.uniform(0, 10, n), rng.uniform(0, 10, n), rng.uniform(0, 1, len(af))
    L, gx, gy = G.timing_loss(x, y, w, 1.0)
    Lo, ox, oy = oracle.timing_loss(g, x.astype(np.float32), y.astype(np.float32), w.astype(np.float32), 1.0)
    assert np.allclose(gx.cpu().numpy(), ox, rtol=1e-5, atol=1e-5)
    G.close()
    _ = src
