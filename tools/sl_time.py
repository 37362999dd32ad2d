"""Time the sweep kernels (schedule 0) at a config: fwd/bwd per pass (CUDA events), the cone
pass on 1% sizing steps, optional per-barrier trace (INSTA_SL_TRACE=dir).
  python tools/sl_time.py C4 [tau] [schedule]"""
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
sched = int(sys.argv[3]) if len(sys.argv) > 3 else 0
g = synth.generate(cfg)
G = insta.Graph(g)
st = torch.cuda.Stream()
dm = torch.empty((g.num_arcs, 2), dtype=torch.float32, device="cuda")
trace = os.environ.pop("INSTA_SL_TRACE", None)
with torch.cuda.stream(st):
    for _ in range(3):
        G.forward(3.0, tau, sched, sync=False, stream=st)
        G.backward(out=dm, stream=st)
    st.synchronize()
    f, b = [], []
    for _ in range(10):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record(st)
        G.forward(3.0, tau, sched, sync=False, stream=st)
        e[1].record(st)
        G.backward(out=dm, stream=st)
        e[2].record(st)
        st.synchronize()
        f.append(e[0].elapsed_time(e[1]))
        b.append(e[1].elapsed_time(e[2]))
    print(f"{cfg} tau={tau} sched={sched}: fwd {np.median(f):.4f} ms  bwd {np.median(b):.4f} ms", flush=True)
    if trace:
        os.environ["INSTA_SL_TRACE"] = trace
        G.forward(3.0, tau, sched, sync=False, stream=st)
        G.backward(out=dm, stream=st)
        st.synchronize()
        os.environ.pop("INSTA_SL_TRACE")
        for name in ("fwd", "bwd", "fwd_lse", "bwd_lse"):
            p = os.path.join(trace, f"sl_{name}.bin")
            if os.path.exists(p):
                raw = np.fromfile(p, np.uint64).astype(np.int64)
                t = raw[:512]
                t = t[t > 0]
                if t.size == 0:
                    continue
                d = np.diff(t) / 1e3
                print(name, "total us", (t[-1] - t[0]) / 1e3, "per barrier us:", " ".join(f"{x:.1f}" for x in d))
                arr = raw[512:]
                nb = len(t)
                grid = len(arr) // (nb + 8) // 2 if nb else 0
                if grid:
                    A = arr[: (len(arr) // grid) * grid].reshape(-1, grid)
                    rows = [k for k in range(A.shape[0]) if (A[k] > 0).all()]
                    out = []
                    for k in rows[1:]:
                        prev = t[k - 1] if k - 1 < len(t) else None   # CTA 0's exit of barrier k-1
                        if prev is None:
                            continue
                        a = (A[k] - prev) / 1e3
                        out.append(f"{k}:{a.min():.1f}/{np.median(a):.1f}/{a.max():.1f}")
                    print(name, "arrival after previous exit (min/med/max us):", " ".join(out))
                    # phases (INSTA_SL_PHASES builds): per (level, CTA) {exit, staged, gathered, done}
                    off = (nb + 8) * 2 * grid if False else None
                    L = (len(arr) // grid) // 6 - 8
                    ph = raw[512 + (L + 8) * 2 * grid: 512 + (L + 8) * 2 * grid + L * grid * 4].reshape(L, grid, 4)
                    if (ph[1:, :, 0] > 0).any():
                        outp = []
                        for s_ in range(1, L):
                            p4 = ph[s_].astype(np.int64)
                            ok = (p4 > 0).all(axis=1)
                            if not ok.any():
                                continue
                            p4 = p4[ok]
                            d = np.diff(p4, axis=1) / 1e3
                            outp.append(f"{s_}:" + "/".join(f"{np.median(d[:, i]):.2f}" for i in range(3)) + f"(max {d.sum(axis=1).max():.1f})")
                        print(name, "phases median us (stage wait / gathers / rest of work):", " ".join(outp))
    # cone pass: 1% sizing steps
    ts, cone = [], []
    for k in range(6):
        ids, m, s = synth.sizing_step(g, k, frac=0.01)
        ids, m, s = (torch.as_tensor(x, device="cuda") for x in (ids, m, s))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        G.update_arcs(ids, m, s, incremental=True, stream=st)
        G.forward(3.0, tau, sched, sync=False, stream=st)
        e1.record(st)
        st.synchronize()
        ts.append(e0.elapsed_time(e1))
        cone.append(G.last_forward_stats() / g.num_pins)
    print("cone ms", " ".join(f"{x:.3f}" for x in ts), "pins frac", " ".join(f"{x:.3f}" for x in cone), flush=True)
    for frac in (1e-7, 1e-5, 1e-4, 1e-3):   # small updates: 1 cell, ~1e-5 of the arcs, ...
        ts, cone = [], []
        for k in range(5):
            ids, m, s = synth.sizing_step(g, 100 + k, frac=frac)
            ids, m, s = (torch.as_tensor(x, device="cuda") for x in (ids, m, s))
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            G.update_arcs(ids, m, s, incremental=True, stream=st)
            G.forward(3.0, tau, sched, sync=False, stream=st)
            e1.record(st)
            st.synchronize()
            ts.append(e0.elapsed_time(e1))
            cone.append(G.last_forward_stats() / g.num_pins)
        print(f"update frac {frac:g} ({len(ids)} arcs): ms", " ".join(f"{x:.3f}" for x in ts), "pins frac",
              " ".join(f"{x:.4f}" for x in cone), flush=True)
    if trace:   # one more cone pass, traced
        ids, m, s = synth.sizing_step(g, 9, frac=0.01)
        ids, m, s = (torch.as_tensor(x, device="cuda") for x in (ids, m, s))
        G.update_arcs(ids, m, s, incremental=True, stream=st)
        st.synchronize()
        os.environ["INSTA_SL_TRACE"] = trace
        t0 = time.perf_counter()
        G.forward(3.0, tau, sched, sync=False, stream=st)
        st.synchronize()
        os.environ.pop("INSTA_SL_TRACE")
        p = os.path.join(trace, "sl_cone.bin")
        if os.path.exists(p):
            raw = np.fromfile(p, np.uint64).astype(np.int64)
            t = raw[:512]
            t = t[t > 0]
            grid = 148
            Lc = (len(raw) - 512) // grid // 10 - 8
            ph = raw[512 + (Lc + 8) * 2 * grid: 512 + (Lc + 8) * 2 * grid + Lc * grid * 8].reshape(Lc, grid, 8)
            if (ph[:, :, 0] > 0).any():
                out = []
                for s_ in range(1, Lc):
                    p8 = ph[s_].astype(np.int64)
                    ok = p8[:, 0] > 0
                    if not ok.any():
                        continue
                    p8 = p8[ok]
                    base = p8[:, 0:1]
                    rel = np.where(p8 > 0, (p8 - base) / 1e3, np.nan)
                    med = np.nanmedian(rel, axis=0)
                    mx = np.nanmax(rel, axis=0)
                    out.append(f"{s_}:" + "/".join("-" if np.isnan(v) else f"{v:.1f}" for v in med[1:7]) +
                               f"(max {np.nanmax(mx):.1f})")
                print("cone phases rel. to barrier exit, median us (flag/stage/-/gath/loop/flush):", " ".join(out[:30]))
            print("cone total us", (t[-1] - t[0]) / 1e3, "barriers", len(t) - 1, "per barrier us:",
                  " ".join(f"{x:.1f}" for x in np.diff(t) / 1e3))
G.close()
