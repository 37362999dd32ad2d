"""Per-level latency vs level width on synthetic layered graphs (debug).

Level l has W pins; every pin of level l > 0 has `fanin` arcs from random pins
of level l-1.  Reports forward / backward time per level for each width.
"""
import os
import sys
import types

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402


def layered(W, L, fanin, seed=0):
    rng = np.random.default_rng(seed)
    N = W * L
    sink = np.repeat(np.arange(W, N), fanin)
    lvl = sink // W
    src = (lvl - 1) * W + rng.integers(0, W, sink.size)
    E = sink.size
    return types.SimpleNamespace(
        num_pins=N, arc_from=src.astype(np.int32), arc_to=sink.astype(np.int32),
        arc_unate=rng.integers(0, 3, E).astype(np.uint8), arc_class=None,
        arc_mean=rng.uniform(1, 10, (E, 2)).astype(np.float32), arc_sigma=rng.uniform(0, 1, (E, 2)).astype(np.float32),
        src_mean=np.zeros((N, 2), np.float32), src_sigma=np.ones((N, 2), np.float32),
        ep_pin=np.arange((L - 1) * W, N, dtype=np.int32), ep_rat=np.full((W, 2), 100.0, np.float32))


def timeit(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1e3   # us


L = int(os.environ.get("LEVELS", "160"))
FANINS = [int(x) for x in os.environ.get("FANINS", "1,2").split(",")]
WIDTHS = [int(x) for x in os.environ.get("WIDTHS", "1,16,148,1024,8192,32768,65536").split(",")]
for fanin in FANINS:
    for W in WIDTHS:
        g = layered(W, L, fanin)
        G = insta.Graph(g)
        d = torch.empty((g.arc_from.size, 2), device="cuda")
        tf = timeit(lambda: G.forward(3.0, 0.0, sync=False))
        tb = timeit(lambda: G.backward(out=d))
        print(f"fanin {fanin} W {W:6d}: fwd {tf:8.1f} us ({tf / L:6.2f} us/level)  bwd {tb:8.1f} us ({tb / L:6.2f} us/level)",
              flush=True)
        G.close()
