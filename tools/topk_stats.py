"""Survivor histogram of the Top-K merge (needs a -DTK_STATS build; INSTA_ROOT points at it)."""
import ctypes
import os
import sys

ROOT = os.environ.get("INSTA_ROOT") or os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

g = synth.generate(sys.argv[1] if len(sys.argv) > 1 else "C4")
G = insta.Graph(g)
G.topk_forward(int(sys.argv[2]) if len(sys.argv) > 2 else 32, 3.0)
import torch  # noqa: E402
torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * 33)()
lib = insta._capi.load()
print("rc", lib.insta_debug_topk_stats(buf))
tot = sum(buf)
print("batches", tot, [(k, buf[k], round(buf[k] / max(tot, 1), 4)) for k in range(33) if buf[k]])
