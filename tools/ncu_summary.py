"""Summary of one kernel in an ncu report: duration, DRAM, occupancy, issue, stall mix and the
hottest SASS lines.   python tools/ncu_summary.py rep.ncu-rep [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 20
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, v = r[0], r[2]
def g(name):
    return v[h.index(name)] if name in h else "?"
for m in ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
          "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
          "smsp__inst_executed.sum", "sm__inst_executed.avg.per_cycle_active", "lts__t_sector_hit_rate.pct"]:
    print(f"{m}: {g(m)}")
st = [(h[i], float(v[i].replace(",", ""))) for i in range(len(h))
      if h[i].startswith("smsp__pcsamp_warps_issue_stalled") and not h[i].endswith("not_issued")
      and v[i].replace(",", "").replace(".", "").isdigit()]
tot = sum(x for _, x in st) or 1
print("stalls:", ", ".join(f"{a.split('stalled_')[1]} {100 * b / tot:.0f}%" for a, b in sorted(st, key=lambda x: -x[1])[:8]))
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hh = rows[1]
rows = rows[2:]
i_s, i_src, i_a = hh.index("Warp Stall Sampling (All Samples)"), hh.index("Source"), hh.index("Address")
i_e = hh.index("Instructions Executed")
tot = sum(float(x[i_s] or 0) for x in rows) or 1
print("total sampled", tot, "instructions executed", sum(float(x[i_e] or 0) for x in rows))
addr = [x[i_a] for x in rows]
for x in sorted(rows, key=lambda x: -float(x[i_s] or 0))[:top]:
    k = addr.index(x[i_a])
    prev = rows[k - 1][i_src].strip()[:50] if k else ""
    print(f"{100 * float(x[i_s]) / tot:5.1f}%  {x[i_src].strip()[:60]:60s} <- {prev}")
