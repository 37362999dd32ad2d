"""Top-K (NEXT 1) timing on a config: insta_topk_forward + insta_topk_slack per K, CUDA events.

    python tools/topk_bench.py [C4] [K ...]
"""
import json
import os
import sys

ROOT = os.environ.get("INSTA_ROOT") or os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
Ks = [int(x) for x in sys.argv[2:]] or [1, 8, 32]
g = synth.generate(cfg)
G = insta.Graph(g)
G.set_cppr_rat(*synth.cppr_rat_table(g))
st = torch.cuda.Stream()
out = []
for K in Ks:
    with torch.cuda.stream(st):
        for _ in range(2):
            G.topk_forward(K, 3.0, stream=st)
            G.topk_slack(stream=st, sync=False)
        st.synchronize()
        n = 5
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        ev[0].record(st)
        for _ in range(n):
            G.topk_forward(K, 3.0, stream=st)
        ev[1].record(st)
        for _ in range(n):
            G.topk_slack(stream=st, sync=False)
        ev[2].record(st)
        st.synchronize()
        summ, _, _ = G.topk_slack(stream=st)
    f_ms = ev[0].elapsed_time(ev[1]) / n
    s_ms = ev[1].elapsed_time(ev[2]) / n
    out.append(dict(config=cfg, K=K, fwd_ms=f_ms, slack_ms=s_ms, tns=summ.tns, wns=summ.wns,
                    nviol=summ.num_violations, pins=g.num_pins, arcs=g.num_arcs))
    out[-1]["variant"] = os.environ.get("VARIANT", "")
    print(json.dumps(out[-1]), flush=True)
G.close()
