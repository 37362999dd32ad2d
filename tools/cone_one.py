"""One-cell incremental updates at C4 (for an ncu launch list of the cone pass)."""
import os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth
g = synth.generate(sys.argv[1] if len(sys.argv) > 1 else "C4")
G = insta.Graph(g)
G.forward(3.0, 0.0)
for k in range(4):
    ids, m, s = synth.sizing_step(g, 100 + k, frac=1e-7)
    G.update_arcs(ids, m, s, incremental=True)
    G.forward(3.0, 0.0)
torch.cuda.synchronize()
print("done", G.last_forward_stats())
