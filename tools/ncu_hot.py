"""Summarize an ncu source page (SASS) csv: top instructions by stall samples and stall totals."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = rows[2:]
ai, si, ni = hdr.index("Address"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
tot = {hdr[i]: 0 for i in stall_cols}
samples = []
for r in data:
    if len(r) != len(hdr):
        continue
    try:
        n = int(r[ni] or 0)
    except ValueError:
        continue
    samples.append((n, r[ai], r[si], {hdr[i]: int(r[i] or 0) for i in stall_cols}))
    for i in stall_cols:
        tot[hdr[i]] += int(r[i] or 0)
S = sum(s[0] for s in samples)
print("total samples", S)
for k, v in sorted(tot.items(), key=lambda x: -x[1])[:8]:
    print(f"  {k:28s} {v:8d} {100*v/max(S,1):5.1f}%")
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
for n, a, s, st in sorted(samples, key=lambda x: -x[0])[:top]:
    main = sorted(st.items(), key=lambda x: -x[1])[:2]
    print(f"{n:7d} {100*n/max(S,1):5.1f}% {a} {s[:70]:70s} {main}")
