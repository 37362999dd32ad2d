"""Replicates csrc/items.cpp on the host to report item/round counts per config."""
import os
import sys
import numpy as np
sys.path.insert(0, '.')
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth

def rounds(prefix_w, pins_cnt, arcs_cnt, fo_cnt, G, caps):
    lo_n = len(prefix_w) - 1
    m = 1
    while True:
        n = m * G
        W = prefix_w[-1]
        cuts = [0] + [int(np.searchsorted(prefix_w, (j * W + n - 1) // n)) for j in range(1, n)] + [lo_n]
        cuts = np.maximum.accumulate(np.minimum(cuts, lo_n))
        ok = True
        for j in range(n):
            a, b = cuts[j], cuts[j + 1]
            if b - a <= 1: continue
            if b - a > caps[0] or arcs_cnt[b] - arcs_cnt[a] > caps[1] or fo_cnt[b] - fo_cnt[a] > caps[2]:
                ok = False; break
        if ok or n >= lo_n: return m
        m *= 2

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
G = 148
g = synth.generate(cfg)
lv = insta.levelize(g.num_pins, g.arc_from, g.arc_to)
fi = np.diff(lv["fanin_ptr"])
fo_full = np.diff(lv["fanout_ptr"])
lfo = np.where(fo_full > 256, 0, fo_full)
level = lv["level"][lv["order"]]
lp = np.searchsorted(level, np.arange(lv["num_levels"] + 1))
tf = tb = 0
widths = []
for l in range(lv["num_levels"]):
    a, b = lp[l], lp[l + 1]
    f = fi[a:b]; o = lfo[a:b]
    pc = np.concatenate([[0], np.cumsum(f)])
    oc = np.concatenate([[0], np.cumsum(o)])
    wf = np.concatenate([[0], np.cumsum(1 + f)])
    wb = np.concatenate([[0], np.cumsum(1 + f + o)])
    rf = rounds(wf, None, pc, np.zeros_like(pc), G, (2048, 2560, 1 << 30))
    rb = rounds(wb, None, pc, oc, G, tuple(int(x) for x in os.environ.get("BWD_CAPS", "1024,2048,2048").split(",")))
    tf += rf; tb += rb
    widths.append((b - a, int(pc[-1]), rf, rb))
print("levels", lv["num_levels"], "fwd steps", tf, "bwd steps", tb)
print("first levels (pins, arcs, fwd rounds, bwd rounds):", widths[:12])
print("median pins/level", int(np.median([w[0] for w in widths])))
