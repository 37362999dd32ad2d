"""Cone-pass probe: per update size, CUDA-event time of insta_update_arcs and of the cone
forward alone (forced: cone_max huge), pins recomputed, and (INSTA_SL_TRACE=dir) the
per-barrier trace of one cone pass.
  python tools/cone_probe.py C4 1e-7 1e-5 1e-3 0.01"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_dac_lugklr25_b200 as insta  # noqa: E402
from paper_conf_dac_lugklr25_b200 import synth  # noqa: E402

cfg = sys.argv[1]
fracs = [float(x) for x in sys.argv[2:]] or [1e-7, 1e-5, 1e-3, 1e-2]
g = synth.generate(cfg)
G = insta.Graph(g)
st = torch.cuda.Stream()
trace = os.environ.pop("INSTA_SL_TRACE", None)
with torch.cuda.stream(st):
    G.forward(3.0, 0.0, 0, sync=False, stream=st)
    for _ in range(3):
        G.forward(3.0, 0.0, 0, sync=False, stream=st)
    st.synchronize()
    e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    e[0].record(st)
    G.forward(3.0, 0.0, 0, sync=False, stream=st)
    e[1].record(st)
    st.synchronize()
    print(f"{cfg}: full forward {e[0].elapsed_time(e[1]):.4f} ms", flush=True)
    for frac in fracs:
        tu, tf, cone = [], [], []
        for k in range(6):
            ids, m, s = synth.sizing_step(g, 200 + k, frac=frac)
            ids, m, s = (torch.as_tensor(x, device="cuda") for x in (ids, m, s))
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
            ev[0].record(st)
            G.update_arcs(ids, m, s, incremental=True, stream=st)
            ev[1].record(st)
            G.forward(3.0, 0.0, 0, sync=False, stream=st, cone_max=10 ** 12)
            ev[2].record(st)
            st.synchronize()
            tu.append(ev[0].elapsed_time(ev[1]))
            tf.append(ev[1].elapsed_time(ev[2]))
            cone.append(G.last_forward_stats() / g.num_pins)
        print(f"frac {frac:g} ({len(ids)} arcs): update ms {np.median(tu):.4f}  cone fwd ms {np.median(tf):.4f} "
              f"(min {min(tf):.4f})  pins frac {np.median(cone):.2e}", flush=True)
        if trace:
            ids, m, s = synth.sizing_step(g, 300, frac=frac)
            ids, m, s = (torch.as_tensor(x, device="cuda") for x in (ids, m, s))
            G.update_arcs(ids, m, s, incremental=True, stream=st)
            st.synchronize()
            os.environ["INSTA_SL_TRACE"] = trace
            G.forward(3.0, 0.0, 0, sync=False, stream=st, cone_max=10 ** 12)
            st.synchronize()
            os.environ.pop("INSTA_SL_TRACE")
            p = os.path.join(trace, "sl_cone.bin")
            if os.path.exists(p):
                raw = np.fromfile(p, np.uint64).astype(np.int64)
                t = raw[:512]
                t = t[t > 0]
                print("  trace: total us", (t[-1] - t[0]) / 1e3, "barriers", len(t) - 1, "per barrier us:",
                      " ".join(f"{x:.1f}" for x in np.diff(t) / 1e3), flush=True)
                grid = G.schedule_info().get("sl_grid", 148) if hasattr(G, "schedule_info") else 148
                nb = 512
                Lc = (len(raw) - 512) // grid // 10 - 8
                if Lc > 0:
                    ph = raw[512 + (Lc + 8) * 2 * grid: 512 + (Lc + 8) * 2 * grid + Lc * grid * 8]
                    if len(ph) == Lc * grid * 8:
                        ph = ph.reshape(Lc, grid, 8)
                        out = []
                        for s_ in range(1, Lc):
                            p8 = ph[s_].astype(np.int64)
                            ok = p8[:, 0] > 0
                            if not ok.any():
                                continue
                            p8 = p8[ok]
                            rel = np.where(p8 > 0, (p8 - p8[:, 0:1]) / 1e3, np.nan)
                            med = np.nanmedian(rel, axis=0)
                            mx = np.nanmax(rel, axis=0)
                            out.append(f"{s_}:" + "/".join("-" if np.isnan(v) else f"{v:.1f}" for v in med[1:7]) +
                                       f"(max {np.nanmax(mx):.1f})")
                        if out:
                            print("  phases rel. to level start, median us (flag/stage/-/gath/loop/flush):",
                                  " ".join(out), flush=True)
G.close()
