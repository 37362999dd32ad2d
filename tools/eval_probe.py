"""insta_eval_candidates probe: device time per candidate (CUDA events around the packed call) and the
per-barrier trace of one small call (INSTA_SL_TRACE=dir).  python tools/eval_probe.py C4 [n]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 512
g = synth.generate(cfg)
G = insta.Graph(g)
st = torch.cuda.Stream()
trace = os.environ.pop("INSTA_SL_TRACE", None)
scs = [synth.sizing_scenario(g, s) for s in range(512, 512 + n)]
with torch.cuda.stream(st):
    G.forward(3.0, 0.0, stream=st)
    pk = G.pack_candidates(scs, stream=st)
    G.eval_packed(pk, stream=st)
    st.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    out = G.eval_packed(pk, stream=st)
    e1.record(st)
    st.synchronize()
    ms = e0.elapsed_time(e1)
    print(f"{cfg}: {n} candidates in {ms:.3f} ms = {1e3 * ms / n:.1f} us each ({n / (ms * 1e-3):.0f} evals/s); "
          f"arcs per candidate {np.mean([len(s['delta_arc']) for s in scs]):.1f}", flush=True)
    if trace:
        small = G.pack_candidates(scs[:8], stream=st)
        os.environ["INSTA_SL_TRACE"] = trace
        G.eval_packed(small, stream=st)
        st.synchronize()
        os.environ.pop("INSTA_SL_TRACE")
        raw = np.fromfile(os.path.join(trace, "sl_eval.bin"), np.uint64).astype(np.int64)
        t = raw[:512]
        t = t[t > 0]
        print("trace (8 candidates): total us", (t[-1] - t[0]) / 1e3, "barriers", len(t) - 1, "per barrier us:",
              " ".join(f"{x:.1f}" for x in np.diff(t) / 1e3), flush=True)
G.close()
