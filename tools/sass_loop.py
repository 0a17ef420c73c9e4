"""Offline look at the hot loop of a JIT module (no GPU): after tools/jit_sass.py
has written /tmp/jit_sass/k.{cu,sass}, split the kern_*_inj function's SASS into
basic blocks and print the blocks that hold SASS of the full-warp self-loop's
first unrolled copy (generated-source lines [first, U<L>_)), with their sizes,
successors and opcode mix — the FFMA blocks and the paths between them are the
hot loop.  usage: sass_loop.py [-v]"""
import collections
import re
import sys

src = open("/tmp/jit_sass/k.cu").read().splitlines()
lo = next(i for i, l in enumerate(src, 1) if "full warp, two iterations per trip" in l)
hi = next(i for i, l in enumerate(src, 1) if i > lo and re.match(r"\s*U\d+_(\d+)?: ;", l))
hi2 = next(i for i, l in enumerate(src, 1) if i > hi and "self-loop" in l)
rows, cur, label = [], None, None
for line in open("/tmp/jit_sass/k.sass"):
    m = re.search(r'//## File "([^"]+)", line (\d+)', line)
    if m:
        cur = int(m.group(2))
        continue
    m = re.match(r"\s*(\.L_x_\d+):", line)
    if m:
        label = m.group(1)
        rows.append(("L", label, cur))
        continue
    m = re.search(r"/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if m:
        rows.append(("I", m.group(2).strip(), cur))
blocks, b = [], None
for kind, txt, ln in rows:
    if kind == "L" or b is None:
        b = {"label": txt if kind == "L" else "entry", "ins": [], "succ": []}
        blocks.append(b)
        if kind == "L":
            continue
    b["ins"].append((txt, ln))
    t = re.search(r"`\((\.L_x_\d+)\)", txt)
    if t and ("BRA" in txt or "BREAK" in txt or "SSY" in txt):
        b["succ"].append(t.group(1))
    if re.match(r"^(@!?U?P\w+\s+)?(BRA|EXIT|RET|BREAK)", txt) or txt.startswith("BRA "):
        b = {"label": "", "ins": [], "succ": []}
        blocks.append(b)


def part(ln):
    return "A" if ln and lo <= ln < hi else ("B" if ln and hi <= ln < hi2 else "-")


tot = collections.Counter()
for k, b in enumerate(blocks):
    where = collections.Counter(part(ln) for _, ln in b["ins"])
    if not where["A"]:
        continue
    ops = collections.Counter(re.sub(r"^@!?U?P\w+\s+", "", t).split()[0] for t, _ in b["ins"])
    ffma = ops.get("FFMA", 0)
    print(f"#{k} {b['label']:>10} n={len(b['ins']):3d} ffma={ffma:2d} succ={b['succ']} "
          + ", ".join(f"{o} {c}" for o, c in ops.most_common(12) if o != "FFMA"))
    if "-v" in sys.argv:
        for t, ln in b["ins"]:
            if not t.startswith("FFMA"):
                print(f"      {ln:5d} {t}")
print(f"copy A: source lines {lo}..{hi - 1}")
