"""Exercise every kernel family on a small graph (compute-sanitizer target):
schedules 0-3 fwd/bwd (hard, LSE), sigma channel, cone pass, eval_candidates,
batched scenarios, Top-K, Clark, Eq 7/8, INSTA-Size steps."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth

cfg = sys.argv[1] if len(sys.argv) > 1 else "C1"
g = synth.generate(cfg)
G = insta.Graph(g)
for tau in (0.0, 1.0):
    for sched in (0, 1, 2, 3):
        G.forward(3.0, tau, sched)
        G.backward()
        G.arrivals()
    G.forward(3.0, tau, 0)
    G.backward(want_src=True, want_sigma=True)
    ids, m, s = synth.sizing_step(g, 1, frac=1e-4)
    G.update_arcs(ids, m, s, incremental=True)
    G.forward(3.0, tau, 0, cone_max=10 ** 9)
    G.backward()
    G.eval_candidates([synth.sizing_scenario(g, k) for k in range(512, 516)])
    scs = [dict(n_sigma=3.0, derate_cell=1.02, derate_net=0.99)] + [synth.sizing_scenario(g, 600 + k) for k in range(3)]
    G.forward_batch(scs, tau=tau, want_grad=True)
G.set_cppr_rat(*synth.cppr_rat_table(g))
G.topk_forward(4, 3.0)
G.topk_slack()
G.clark_forward(3.0)
G.clark_backward(want_sigma=True)
G.forward(3.0, 0.0)
d = G.backward()
w = -(d[:, 0] + d[:, 1])
rng = np.random.default_rng(1)
L, gx, gy = G.timing_loss(rng.uniform(0, 100, g.num_pins), rng.uniform(0, 100, g.num_pins), w, 1e-3)
r = insta.grad_norm_ratio(torch.rand(100, device="cuda"), torch.rand(100, device="cuda"))
sg = G.stage_gradients(d)
G.select_stages(sg, 0.0)
torch.cuda.synchronize()
print("ok", float(r.item()))
G.close()
