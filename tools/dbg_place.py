import numpy as np, torch, sys
sys.path.insert(0, '/root/repo')
import oracle, paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth
g = synth.generate("C2")
rng = np.random.default_rng(11)
x = rng.uniform(0, 1000, g.num_pins).astype(np.float32)
y = rng.uniform(0, 1000, g.num_pins).astype(np.float32)
for sched in (0, 2):
    G = insta.Graph(g)
    G.forward(3.0, 0.0, sched)
    d = G.backward()
    w = -(d[:, 0] + d[:, 1])
    L, gx, gy = G.timing_loss(x, y, w, lambda_rc=1e-3)
    L2, _, _ = G.timing_loss(x, y, w.cpu().numpy().copy(), lambda_rc=1e-3)
    torch.cuda.synchronize()
    print(sched, float(L.item()), float(L2.item()), float(w.sum()), int((w > 0).sum()))
    Lo, _, _ = oracle.timing_loss(g, x, y, w.cpu().numpy(), float(np.float32(1e-3)))
    print("oracle", Lo)
    G.close()
