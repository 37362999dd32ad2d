"""Per-item timeline of the persistent kernels (debug; run on the GPU box).

Runs C4 forward+backward a few times, then once with INSTA_TRACE_DIR set, and
summarizes the globaltimer stamps each worker warp recorded per item step.
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
tau = float(sys.argv[2]) if len(sys.argv) > 2 else 0.0
out = os.environ.get("OUT", "gpurun_out")
g = synth.generate(cfg)
G = insta.Graph(g)
for _ in range(3):
    G.forward(3.0, tau, sync=False)
    G.backward()
torch.cuda.synchronize()
if os.environ.get("INC"):   # trace an incremental forward after a 1 % sizing step
    ids, m, s_ = synth.sizing_step(g, 0, frac=0.01)
    G.update_arcs(ids, m, s_, incremental=True)
    torch.cuda.synchronize()
os.environ["INSTA_TRACE_DIR"] = out
G.forward(3.0, tau, sync=False)
G.backward()
torch.cuda.synchronize()
del os.environ["INSTA_TRACE_DIR"]


def load(name):
    raw = open(os.path.join(out, name), "rb").read()
    grid, steps, k = np.frombuffer(raw[:12], np.int32)
    return np.frombuffer(raw[12:], np.uint64).reshape(grid, steps, k).astype(np.int64)


for name in ("fwd_trace.bin", "bwd_trace.bin"):
    t = load(name)
    t0 = t[:, 0, 0].min()
    s0, s1, s2 = (t[..., i] - t0 for i in range(3))   # item start, gathers done, item done
    has_g = t[..., 1] > 0
    if not has_g.any():   # kernels that stamp only start/end (warp-independent forward)
        s1 = s0
        has_g = t[..., 2] > 0
    print(f"== {name}: grid={t.shape[0]} steps={t.shape[1]} total={s2.max()/1e3:.1f} us")
    gather = np.where(has_g, s1 - s0, 0)
    comp = np.where(has_g, s2 - s1, 0)
    print("  per item: gather phase median %.2f us (p99 %.2f), compute phase median %.2f us (p99 %.2f)" % (
        np.median(gather[has_g]) / 1e3, np.percentile(gather[has_g], 99) / 1e3,
        np.median(comp[has_g]) / 1e3, np.percentile(comp[has_g], 99) / 1e3))
    s3 = t[..., 3] - t0
    has3 = has_g & (t[..., 3] > 0)
    if has3.any():   # forward: slot 3 = stale words re-polled and folded pins computed
        poll = np.where(has3, s3 - s1, 0)
        rnd = np.where(has3, s2 - s3, 0)
        print("  forward split: poll+fold median %.2f us (p90 %.2f), rounds median %.2f us (p90 %.2f)" % (
            np.median(poll[has3]) / 1e3, np.percentile(poll[has3], 90) / 1e3,
            np.median(rnd[has3]) / 1e3, np.percentile(rnd[has3], 90) / 1e3))
    end_max = s2.max(axis=0)
    start_min = s0.min(axis=0)
    inc = np.diff(np.concatenate([[0], end_max]))
    print("  step completion increment: median %.2f us, mean %.2f us" % (np.median(inc) / 1e3, inc.mean() / 1e3))
    for k in list(range(0, 10)) + list(range(t.shape[1] // 2, t.shape[1] // 2 + 4)) + list(range(t.shape[1] - 4, t.shape[1])):
        gk = gather[:, k][has_g[:, k]]
        ck = comp[:, k][has_g[:, k]]
        print(f"  step {k:4d}: start[min {start_min[k]/1e3:8.1f}] end[max {end_max[k]/1e3:8.1f}] inc {inc[k]/1e3:6.2f}"
              f" | gather med {np.median(gk)/1e3 if gk.size else 0:5.2f} max {gk.max()/1e3 if gk.size else 0:5.2f}"
              f" | compute med {np.median(ck)/1e3 if ck.size else 0:5.2f} max {ck.max()/1e3 if ck.size else 0:5.2f}")

# per-level view of the forward: step increments next to the level sizes
if os.environ.get("LEVELS_VIEW"):
    lv = insta.levelize(g.num_pins, g.arc_from, g.arc_to)
    level = np.asarray(lv["level"])
    sizes = np.bincount(level)
    print("level sizes (pins):", " ".join(str(x) for x in sizes))
    t = load("fwd_trace.bin")
    t0 = t[:, 0, 0].min()
    end_max = (t[..., 2] - t0).max(axis=0)
    inc = np.diff(np.concatenate([[0], end_max]))
    print("fwd step increments (us):", " ".join(f"{x/1e3:.1f}" for x in inc))

# per-step spread of item completion (relative to the previous step's last end)
if os.environ.get("SPREAD"):
    for name in ("fwd_trace.bin", "bwd_trace.bin"):
        t = load(name)
        t0 = t[:, 0, 0].min()
        st, en = t[..., 0] - t0, t[..., 2] - t0
        prev = 0
        print("==", name)
        lo, hi = (int(x) for x in os.environ["SPREAD"].split(":"))
        for s in range(t.shape[1]):
            a, b = st[:, s], en[:, s]
            ok = b > 0
            a, b = a[ok], b[ok]
            if a.size and lo <= s < hi:
                print(f"step {s:3d}: n={a.size:3d} start rel [min {(a.min()-prev)/1e3:6.2f} med {(np.median(a)-prev)/1e3:6.2f}]"
                      f" end rel [min {(b.min()-prev)/1e3:6.2f} med {(np.median(b)-prev)/1e3:6.2f} p90 {(np.percentile(b,90)-prev)/1e3:6.2f} max {(b.max()-prev)/1e3:6.2f}]"
                      f" dur med {np.median(b-a)/1e3:5.2f}")
            if a.size:
                prev = b.max()
