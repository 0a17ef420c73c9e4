"""Attribute ncu per-SASS-instruction metrics to CUDA source lines using
nvdisasm -g line info.  usage: sass_lines.py <ncu sass csv> <nvdisasm -g text> [top]"""
import csv
import re
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
iA, iI = h.index("Address"), h.index("Instructions Executed")
iW = h.index("Warp Stall Sampling (All Samples)")
data = [r for r in rows[2:] if len(r) > iI and r[iI].isdigit()]
base = int(data[0][iA], 16)
loc = {}
cur = None
for line in open(sys.argv[2]):
    m = re.search(r'//## File "([^"]+)", line (\d+)', line)
    if m:
        cur = (m.group(1).split("/")[-1], int(m.group(2)))
        continue
    m = re.search(r"/\*([0-9a-f]{4,})\*/", line)
    if m and cur:
        loc[int(m.group(1), 16)] = cur
agg = defaultdict(lambda: [0, 0])
for r in data:
    off = int(r[iA], 16) - base
    k = loc.get(off, ("?", 0))
    agg[k][0] += int(r[iI])
    agg[k][1] += int(r[iW] or 0)
tot = sum(v[0] for v in agg.values())
ts = sum(v[1] for v in agg.values())
src = {}
for k in agg:
    if k[0] != "?" and k[0] not in src:
        try:
            src[k[0]] = open("paper_conf_dsn_0002hsvk21_b200/csrc/" + k[0]).read().split("\n")
        except OSError:
            src[k[0]] = []
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
print("total inst", tot)
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    s = src.get(k[0], [])
    txt = s[k[1] - 1].strip()[:80] if 0 < k[1] <= len(s) else ""
    print(f"{v[0] / tot * 100:5.1f}% stall {v[1] / ts * 100:5.1f}%  {k[0]}:{k[1]}  {txt}")
