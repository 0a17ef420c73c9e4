"""Offline look at the JIT module's code (no GPU): generate the per-program CUDA
for a program (fi_jit_source), compile it with nvcc for sm_100a with the NVRTC
options, and report registers/spills and the static SASS mix of the source
lines of one block.  usage: jit_sass.py [c2|c1|c3|c4] [first_line last_line]"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c2"
mode = int(os.environ.get("MODES", fi.FI_JIT_INJECT))
prog = {"c2": lambda: P.c2(full=False), "c1": P.c1}[name]()
d = "/tmp/jit_sass"
os.makedirs(d, exist_ok=True)
open(f"{d}/k.cu", "w").write(fi.jit_source(prog, mode))
r = subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-cubin", "--fmad=false", "-lineinfo",
                    "-std=c++17", "-Xptxas", "-v", "-o", f"{d}/k.cubin", f"{d}/k.cu"], capture_output=True, text=True)
print("\n".join(l for l in r.stderr.splitlines() if "registers" in l or "spill" in l or "error" in l))
sass = subprocess.run(["nvdisasm", "-g", "-c", f"{d}/k.cubin"], capture_output=True, text=True).stdout
open(f"{d}/k.sass", "w").write(sass)
rows, cur = [], None
for line in sass.splitlines():
    m = re.search(r'//## File "([^"]+)", line (\d+)', line)
    if m:
        cur = int(m.group(2))
        continue
    m = re.search(r"/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if m and cur:
        rows.append((int(m.group(1), 16), cur, m.group(2).strip()))
src = open(f"{d}/k.cu").read().splitlines()
if len(sys.argv) > 3:
    lo, hi = int(sys.argv[2]), int(sys.argv[3])
else:   # the first LDG batch block to the BRA that closes it
    lo = next(i for i, l in enumerate(src, 1) if "LDG batch" in l) - 1
    hi = next(i for i, l in enumerate(src, 1) if i > lo and "exm_ == amask" in l) + 3
sel = [r for r in rows if lo <= r[1] <= hi]
ops = collections.Counter(re.sub(r"^@!?U?P\w+\s+", "", r[2]).split()[0] for r in sel)
print(f"lines {lo}..{hi}: {len(sel)} static SASS;", ", ".join(f"{k} {v}" for k, v in ops.most_common(25)))
print("local memory in the whole module:", sum(1 for r in rows if re.search(r"\b(LDL|STL)", r[2])))
bra = next(i for i, l in enumerate(src, 1) if i > lo and "exm_ == amask" in l) - 1
be = [r for r in rows if r[1] in (bra, bra + 1)]
print(f"back-edge lines {bra},{bra + 1}: {len(be)} static SASS, IMAD.MOV {sum('IMAD.MOV' in r[2] for r in be)}, "
      f"LDL/STL {sum(bool(re.search(r'(LDL|STL)', r[2])) for r in be)}")
