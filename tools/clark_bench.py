"""Clark merge (NEXT 2) timing: insta_clark_forward (+slack) and insta_clark_backward, CUDA events."""
import json
import os
import sys

ROOT = os.environ.get("INSTA_ROOT") or os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
g = synth.generate(cfg)
G = insta.Graph(g)
st = torch.cuda.Stream()
dm = torch.empty((g.num_arcs, 2), dtype=torch.float32, device="cuda")
with torch.cuda.stream(st):
    for _ in range(2):
        G.clark_forward(3.0, sync=False, stream=st)
        G.lib.insta_clark_backward(G._h, None, insta._dptr(dm), None, None, G._st(st))
    st.synchronize()
    n = 5
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    ev[0].record(st)
    for _ in range(n):
        G.clark_forward(3.0, sync=False, stream=st)
    ev[1].record(st)
    for _ in range(n):
        G.lib.insta_clark_backward(G._h, None, insta._dptr(dm), None, None, G._st(st))
    ev[2].record(st)
    st.synchronize()
    s = G.clark_forward(3.0, stream=st)
print(json.dumps(dict(config=cfg, fwd_ms=ev[0].elapsed_time(ev[1]) / n, bwd_ms=ev[1].elapsed_time(ev[2]) / n,
                      tns=s.tns, wns=s.wns, nviol=s.num_violations, pins=g.num_pins)), flush=True)
G.close()
