"""Cone pass vs full pass crossover: update + forward (CUDA events) for sizing updates of several
sizes, the cone pass forced (cone_max huge) and the full pass (incremental=False).
  python tools/cone_cross.py C4"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
g = synth.generate(cfg)
G = insta.Graph(g)
st = torch.cuda.Stream()
with torch.cuda.stream(st):
    G.forward(3.0, 0.0, stream=st)
    for frac in (1e-6, 1e-5, 3e-5, 1e-4, 3e-4, 1e-3):
        res = {}
        upd = [tuple(torch.as_tensor(x, device="cuda") for x in synth.sizing_step(g, 500 + k, frac=frac))
               for k in range(8)]   # generated first: no host gap (idle GPU) inside the timed steps
        for mode in ("cone", "full"):
            ts, fr = [], []
            for k in range(8):
                ids, m, s = upd[k]
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(st)
                G.update_arcs(ids, m, s, incremental=(mode == "cone"), stream=st)
                G.forward(3.0, 0.0, sync=False, stream=st, cone_max=10 ** 12)
                e1.record(st)
                st.synchronize()
                ts.append(e0.elapsed_time(e1))
                fr.append(G.last_forward_stats() / g.num_pins)
            res[mode] = (np.median(ts[1:]), np.median(fr))
        print(f"{cfg} frac {frac:g} ({int(frac * g.num_arcs)} arcs): cone {res['cone'][0]:.3f} ms "
              f"({res['cone'][1]:.4f} pins) full {res['full'][0]:.3f} ms", flush=True)
