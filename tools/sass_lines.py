"""Attribute ncu SASS-level stall samples to CUDA source lines (nvdisasm -g).

usage: python tools/sass_lines.py <ncu source-sass csv> <nvdisasm -g output> <mangled kernel name> [topN]
"""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
import os
ai, ni, si = hdr.index("Address"), hdr.index(os.environ.get("COL", "Warp Stall Sampling (All Samples)")), hdr.index("Source")
data = [r for r in rows[2:] if len(r) == len(hdr)]
base = min(int(r[ai], 16) for r in data)
samples = collections.Counter()
for r in data:
    samples[int(r[ai], 16) - base] += int(r[ni] or 0)
# parse nvdisasm -g for the kernel
lines = open(sys.argv[2]).read().split("\n")
fn = sys.argv[3]
start = None
for idx, l in enumerate(lines):
    if l.strip() == ".text." + fn + ":":
        start = idx
        break
cur = None
off2line = {}
for l in lines[start + 1:]:
    if l.strip().startswith(".section") or (l.strip().endswith(":") and l.strip().startswith(".text.")):
        break
    m = re.search(r'//## File "(.*?)", line (\d+)', l)
    if m:
        cur = (m.group(1), int(m.group(2)))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m and cur is not None:
        off2line[int(m.group(1), 16)] = cur
by_line = collections.Counter()
for off, n in samples.items():
    by_line[off2line.get(off, ("?", -1))] += n
tot = sum(by_line.values())
srcs = {}
top = int(sys.argv[4]) if len(sys.argv) > 4 else 25
for (f, line), n in by_line.most_common(top):
    if f not in srcs:
        try:
            srcs[f] = open(f).read().split("\n")
        except OSError:
            srcs[f] = []
    src = srcs[f]
    text = src[line - 1].strip() if 0 < line <= len(src) else "?"
    print(f"{100 * n / tot:5.1f}%  {f.split('/')[-1]}:{line:<5d} {text[:100]}")
