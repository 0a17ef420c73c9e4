"""Attribute an ncu source page (SASS, --print-source sass --csv) of the JIT
kernel k_inject_jit to lines of the generated CUDA (FI_JIT_DUMP=<p> writes
<p>.cu and <p>.cubin).  usage: jit_lines.py <source.csv> <p> [top]"""
import collections
import csv
import re
import subprocess
import sys

src_csv, dump = sys.argv[1], sys.argv[2]
KERNEL = __import__("os").environ.get("JIT_KERNEL", "k_inject_jit")
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
rows = list(csv.reader(open(src_csv)))
h = rows[1]
iA, iS, iI = h.index("Address"), h.index("Source"), h.index("Instructions Executed")
iW = h.index("Warp Stall Sampling (All Samples)")
data = [r for r in rows[2:] if len(r) > iI]
base = int(data[0][iA], 16)
loc, cur, fn = {}, None, None
for line in subprocess.run(["nvdisasm", "-g", "-c", dump + ".cubin"], capture_output=True, text=True).stdout.splitlines():
    m = re.search(r"\.text\.(\S+):", line)
    if m:
        fn = m.group(1)
    m = re.search(r'//## File "([^"]+)", line (\d+)', line)
    if m:
        cur = int(m.group(2))
        continue
    m = re.search(r"/\*([0-9a-f]{4,})\*/", line)
    if m and cur and fn == KERNEL:
        loc[int(m.group(1), 16)] = cur
src = open(dump + ".cu").read().split("\n")
agg = collections.defaultdict(lambda: [0, 0])
ops = collections.Counter()
for r in data:
    off = int(r[iA], 16) - base
    n, w = int(r[iI] or 0), int(r[iW] or 0)
    agg[loc.get(off, 0)][0] += n
    agg[loc.get(off, 0)][1] += w
    s = r[iS].strip()
    ops[re.sub(r"^@!?U?P\w+\s+", "", s).split()[0] if s else "?"] += n
tot = sum(v[0] for v in agg.values())
ts = sum(v[1] for v in agg.values())
print(f"executed SASS warp-instructions {tot}, stall samples {ts}")
print("by opcode:", ", ".join(f"{k} {v / tot * 100:.1f}%" for k, v in ops.most_common(16)))
print("  inst%  stall%  line of the generated source")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    t = src[k - 1].strip()[:110] if 0 < k <= len(src) else "(no line)"
    print(f"{v[0] / tot * 100:6.1f} {v[1] / ts * 100:6.1f}  L{k}: {t}")
