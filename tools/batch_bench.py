"""Batched scenario throughput on C4 (debug/measurement): evals/s for fwd and fwd+bwd."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
tau = float(sys.argv[2]) if len(sys.argv) > 2 else 0.0
g = synth.generate(cfg)
G = insta.Graph(g)
for B in (32, 64):
    scs = [dict(zip(("n_sigma", "derate_cell", "derate_net"), synth.ocv_scenario(s))) for s in range(B)]
    for grad in (False, True):
        G.forward_batch(scs, tau=tau, want_grad=grad)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 3
        a.record()
        for _ in range(reps):
            G.forward_batch(scs, tau=tau, want_grad=grad)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / reps
        print(f"{cfg} tau={tau} B={B} grad={grad}: {ms:8.2f} ms per batch, {B / ms * 1e3:8.1f} evals/s, "
              f"{B * g.num_pins / ms * 1e3:.3e} pins/s", flush=True)
