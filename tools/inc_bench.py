"""C3 incremental benchmark: per sizing step (1% of arcs), incremental forward vs full forward."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.01
g = synth.generate(cfg)
G = insta.Graph(g)
G.forward(3.0, 0.0)
steps = [synth.sizing_step(g, s, frac=frac) for s in range(6)]
dev = [(torch.as_tensor(i, device="cuda"), torch.as_tensor(m, device="cuda"), torch.as_tensor(s, device="cuda"))
       for i, m, s in steps]
ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
for mode in ("incremental", "full"):
    ts, cones = [], []
    for k, (i, m, s) in enumerate(dev):
        G.update_arcs(i, m, s, incremental=(mode == "incremental"))
        torch.cuda.synchronize()
        a, b = ev(), ev()
        a.record()
        G.forward(3.0, 0.0, sync=False)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
        cones.append(G.last_forward_stats() / g.num_pins)
    print(f"{cfg} {mode:11s}: forward {np.median(ts[1:]) * 1e3:8.1f} us (median of steps 1..5), "
          f"cone {np.median(cones[1:]) * 100:5.1f}% of pins, arcs/step {len(steps[0][0])}")
