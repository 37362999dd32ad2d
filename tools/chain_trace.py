"""Per-step item timing spread on a layered graph (debug; run on the GPU box).

usage: W=65536 FANIN=1 python tools/chain_trace.py   (NO_TRACE=1: just run, e.g. under ncu)
For each step: spread of item start/end times across CTAs relative to the
previous step's last end -- separates dependency jitter from item work.
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


W = int(os.environ.get("W", "65536"))
F = int(os.environ.get("FANIN", "1"))
L = int(os.environ.get("LEVELS", "40"))
out = os.environ.get("OUT", "gpurun_out")
G = insta.Graph(layered(W, L, F))
BWD = bool(os.environ.get("BWD"))
for _ in range(3):
    G.forward(3.0, 0.0, sync=False)
    if BWD:
        G.backward()
torch.cuda.synchronize()
if os.environ.get("NO_TRACE"):   # plain runs only (for ncu captures)
    sys.exit(0)
os.environ["INSTA_TRACE_DIR"] = out
G.forward(3.0, 0.0, sync=False)
if BWD:
    G.backward()
torch.cuda.synchronize()
del os.environ["INSTA_TRACE_DIR"]
raw = open(os.path.join(out, "bwd_trace.bin" if BWD else "fwd_trace.bin"), "rb").read()
grid, steps, k = np.frombuffer(raw[:12], np.int32)
t = np.frombuffer(raw[12:], np.uint64).reshape(grid, steps, k).astype(np.int64)
t0 = t[:, 0, 0].min()
st, en = t[..., 0] - t0, t[..., 2] - t0
g1, g3 = t[..., 1] - t0, t[..., 3] - t0   # warp 0: gathers landed, corners computed (staged rounds)
print(f"W={W} fanin={F} levels={L} grid={grid} steps={steps} total={en.max()/1e3:.1f} us")
prev = 0
for s in range(steps):
    a, b = st[:, s], en[:, s]
    ok = b > 0
    a, b = a[ok], b[ok]
    if not a.size:
        continue
    q = lambda x, p: np.percentile(x, p) / 1e3
    print(f"step {s:3d}: start rel prev-end [min {(a.min()-prev)/1e3:6.2f} med {(np.median(a)-prev)/1e3:6.2f}]"
          f" end rel prev-end [min {(b.min()-prev)/1e3:6.2f} med {(np.median(b)-prev)/1e3:6.2f} p90 {(np.percentile(b,90)-prev)/1e3:6.2f} max {(b.max()-prev)/1e3:6.2f}]"
          f" dur med {np.median(b-a)/1e3:5.2f}", end="")
    m = (t[:, s, 1] > 0) & ok
    if m.any():
        print(f" | w0: landed {np.median(g1[m, s]-prev)/1e3:5.2f} polled+corners {np.median(np.maximum(g3[m, s], 0)-prev)/1e3:5.2f}"
              f" end {np.median(en[m, s]-prev)/1e3:5.2f}", end="")
    print()
    prev = b.max()
