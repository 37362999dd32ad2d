"""Is a full pass slower right after a cone pass?  update(incremental=False) + forward timed
(CUDA events, the stream drained before each step), after full passes and after cone passes."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

g = synth.generate(sys.argv[1] if len(sys.argv) > 1 else "C4")
G = insta.Graph(g)
st = torch.cuda.Stream()
upd = [tuple(torch.as_tensor(x, device="cuda") for x in synth.sizing_step(g, 900 + k, frac=1e-5)) for k in range(24)]


def step(k, inc, time_it=True):
    ids, m, s = upd[k]
    st.synchronize()
    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    e0.record(st)
    G.update_arcs(ids, m, s, incremental=inc, stream=st)
    e1.record(st)
    G.forward(3.0, 0.0, sync=False, stream=st, cone_max=10 ** 12)
    e2.record(st)
    st.synchronize()
    return e0.elapsed_time(e2), e1.elapsed_time(e2)


with torch.cuda.stream(st):
    G.forward(3.0, 0.0, stream=st)
    a = [step(k, False) for k in range(8)]
    b = []
    for k in range(8, 24, 2):
        step(k, True)
        b.append(step(k + 1, False))
    print("full after full : total %.3f ms, forward only %.3f ms" % tuple(np.median(np.array(a[1:]), axis=0)))
    print("full after cone : total %.3f ms, forward only %.3f ms" % tuple(np.median(np.array(b), axis=0)))
