"""Trace one forced cone pass on a 1 % sizing step (phases build + INSTA_SL_TRACE):
per flagged super-level the barrier-to-barrier time and, over CTAs, the median of the phase stamps.
  python tools/cone_trace.py C3 <trace dir>"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg, tdir = sys.argv[1], sys.argv[2]
g = synth.generate(cfg)
G = insta.Graph(g)
G.forward(3.0, 0.0)
for k in range(3):   # warm
    ids, m, s = synth.sizing_step(g, k, frac=0.01)
    G.update_arcs(ids, m, s, incremental=True)
    G.forward(3.0, 0.0, cone_max=10 ** 12)
ids, m, s = synth.sizing_step(g, 9, frac=0.01)
G.update_arcs(ids, m, s, incremental=True)
torch.cuda.synchronize()
os.environ["INSTA_SL_TRACE"] = tdir
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
G.forward(3.0, 0.0, cone_max=10 ** 12)
e1.record()
torch.cuda.synchronize()
print("traced cone pass ms (incl. trace copy):", e0.elapsed_time(e1), "pins frac", G.last_forward_stats() / g.num_pins)
raw = np.fromfile(os.path.join(tdir, "sl_cone.bin"), np.uint64).astype(np.int64)
t = raw[:512]
t = t[t > 0]
grid = 148
Lc = (len(raw) - 512) // grid // 10 - 8
ph = raw[512 + (Lc + 8) * 2 * grid: 512 + (Lc + 8) * 2 * grid + Lc * grid * 8].reshape(Lc, grid, 8)
print("barriers", len(t) - 1, "total us", (t[-1] - t[0]) / 1e3)
print("per barrier us:", " ".join(f"{x:.1f}" for x in np.diff(t) / 1e3))
print("level: median over CTAs of stamps 1..6 relative to stamp 0 (us): flags / stage / first dirty / first gathers / thread0 loop done / CTA flush done / first head done")
for s_ in range(Lc):
    p8 = ph[s_].astype(np.int64)
    ok = p8[:, 0] > 0
    if not ok.any():
        continue
    p8 = p8[ok]
    rel = np.where(p8 > 0, (p8 - p8[:, 0:1]) / 1e3, np.nan)
    med = np.nanmedian(rel, axis=0)
    mx = np.nanmax(rel, axis=0)
    print(f"{s_:3d} " + " ".join("   -  " if np.isnan(v) else f"{v:6.2f}" for v in med[1:8]) + f"   max {np.nanmax(mx):.2f}")
    if s_ in (5, 20, 40):
        slow = np.argsort(-np.nan_to_num(rel[:, 6]))[:3]
        for c in slow:
            print("      slow cta", c, " ".join("   -  " if np.isnan(v) else f"{v:6.2f}" for v in rel[c, 1:8]))
