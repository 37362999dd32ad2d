"""Debug / timing of insta_forward_batch on C4 with per-call synchronization."""
import faulthandler
import os
import sys
import time

ROOT = os.environ.get("INSTA_ROOT") or os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
faulthandler.dump_traceback_later(int(os.environ.get("DUMP_AFTER", "200")), exit=True)

import torch  # noqa: E402

import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
g = synth.generate(cfg)
G = insta.Graph(g)
scs = synth.c5_scenarios(g, n=1024, n_ocv=512)
print("graph ready", insta.__file__, flush=True)
if os.environ.get("FWD_FIRST"):
    print(G.forward(3.0, 0.0), flush=True)
st = torch.cuda.Stream()
for (lo, hi, grad) in [(0, 32, True), (512, 544, False), (0, 512, True), (512, 1024, False), (0, 512, True),
                       (512, 1024, False)]:
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    with torch.cuda.stream(st):
        summ, d = G.forward_batch(scs[lo:hi], want_grad=grad, stream=st)
    t1 = time.perf_counter()
    st.synchronize()
    t2 = time.perf_counter()
    print(f"[{lo},{hi}) grad={grad}: enqueue {1e3*(t1-t0):.1f} ms, total {1e3*(t2-t0):.1f} ms, "
          f"tns[0]={summ[0,1].item():.1f}", flush=True)
G.close()
