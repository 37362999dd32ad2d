"""Per-level phase timestamps of a traced sweep pass (INSTA_SL_PHASES build, INSTA_SL_TRACE dir):
  python tools/phases.py <dir>/sl_fwd.bin [grid]
Per super-level: barrier-to-barrier time (CTA 0), and over CTAs the median / max of
ph[2]-ph[0] (staged slice ready), ph[4]-ph[0] (first head's gathers landed), ph[5]-ph[0] (heads done)."""
import sys
import numpy as np

raw = np.fromfile(sys.argv[1], np.uint64).astype(np.int64)
grid = int(sys.argv[2]) if len(sys.argv) > 2 else 148
t = raw[:512]
t = t[t > 0]
L = (len(raw) - 512) // (10 * grid) - 8
ph = raw[512 + (L + 8) * 2 * grid: 512 + (L + 8) * 2 * grid + L * grid * 8].reshape(L, grid, 8)
bar = np.diff(t) / 1e3 if t.size else np.full(L, np.nan)
if t.size:
    print(f"levels {L}, total {(t[-1] - t[0]) / 1e3:.1f} us")
else:   # no grid barriers (flow mode): level starts per CTA
    st0 = ph[1:, :, 0]
    print(f"levels {L} (no barriers); level start over CTAs relative to the first level (us), median/max:")
    base = st0[0].min()
    print(" ".join(f"{s}:{np.median(st0[s - 1] - base) / 1e3:.1f}/{(st0[s - 1].max() - base) / 1e3:.1f}" for s in range(1, L)))
print("sl  bar_us | stage med/max | gath med/max | done med/max | entries med/max | cta_end med/max (us after barrier exit)")
for s in range(1, L):
    p = ph[s]
    ok = p[:, 0] > 0
    if not ok.any():
        continue
    p = p[ok]
    r = lambda i: (p[:, i] - p[:, 0]) / 1e3
    def mm(i):
        v = r(i)[p[:, i] > 0]
        return f"{np.median(v):5.2f}/{v.max():5.2f}" if v.size else "  -  /  -  "
    b = bar[s - 1] if s - 1 < len(bar) else float("nan")
    ce = ph[s + 1][ok][:, 5] if s + 1 < L else np.zeros(0, np.int64)
    cte = ((ce - p[:, 0]) / 1e3) if ce.size == p.shape[0] else np.zeros(0)
    cts = f"{np.median(cte):5.2f}/{cte.max():5.2f}" if cte.size and (ce > 0).all() else "  -  "
    print(f"{s:3d} {b:6.2f} | {mm(2)} | {mm(4)} | {mm(5)} | {mm(6)} | {cts}")
