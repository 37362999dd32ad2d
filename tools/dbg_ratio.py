import os, sys, types
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth

def ratio(tag):
    a = torch.rand(1000, device="cuda")
    b = torch.rand(1000, device="cuda")
    r = insta.grad_norm_ratio(a, b)
    v1 = float(r.item())
    torch.cuda.synchronize()
    v2 = float(r.item())
    print(tag, v1, v2, float(a.norm() / b.norm()), flush=True)

ratio("start")
g = synth.generate(sys.argv[1] if len(sys.argv) > 1 else "C3")
G = insta.Graph(g)
ratio("after create")
G.forward(3.0, 0.0)
ratio("after forward")
ids, m, s = synth.sizing_step(g, 0, frac=0.01)
G.update_arcs(ids, m, s, incremental=True)
G.forward(3.0, 0.0, cone_max=10 ** 9)
ratio("after cone")
G.backward()
ratio("after backward")
G.close()
ratio("after close")
