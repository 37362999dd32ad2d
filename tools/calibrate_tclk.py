"""Calibrate each config's clock period T_clk (writes nothing; prints the table).

Calls only the oracle (oracle/) and the generator: with T_clk = 0, endpoint
slack is min_rf(off_rf - A_rf) where off_rf is the drawn RAT offset; an
endpoint violates iff T_clk < q = max_rf(A_rf - off_rf).  T_clk is set to the
85th percentile of q (hard mode, N_sigma = 3), so ~15% of endpoints violate
(SURVEY.md §8(d)).  The printed values are pasted into synth.CONFIGS.
"""
import dataclasses
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

for name in sys.argv[1:] or ["C1", "C2", "C3", "C4"]:
    cfg = dataclasses.replace(synth.CONFIGS[name], t_clk=0.0)
    g = synth.generate(cfg)
    A = oracle.forward(g, 3.0, 0.0)["A"][g.ep_pin]
    q = np.max(A - g.ep_rat.astype(np.float64), axis=1)
    print(name, round(float(np.quantile(q, 0.85)), 0), flush=True)
