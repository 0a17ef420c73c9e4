"""The hottest SASS instructions of an ncu source page (--page source --csv
--print-source sass) with their executed counts and stall samples by reason,
in address order, and the kernel's stall totals by reason: where the warps of
k_inject_jit wait.  usage: sass_hot.py <source.csv> [min-exec-fraction]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.002
h = rows[1]
ix = {k: h.index(k) for k in ("Address", "Source", "Instructions Executed", "Warp Stall Sampling (All Samples)")}
reasons = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
data = [r for r in rows[2:] if len(r) > ix["Instructions Executed"]]


def num(x):
    try:
        return float(x.replace(",", ""))
    except ValueError:
        return 0.0


tot_i = sum(num(r[ix["Instructions Executed"]]) for r in data)
tot_s = sum(num(r[ix["Warp Stall Sampling (All Samples)"]]) for r in data)
by = collections.Counter()
for r in data:
    for k in reasons:
        by[k] += num(r[h.index(k)])
print(f"executed {tot_i:.3e}, stall samples {tot_s:.0f}: " +
      ", ".join(f"{k[6:]} {100 * v / tot_s:.1f}%" for k, v in by.most_common(8)))
for r in data:
    e = num(r[ix["Instructions Executed"]])
    s = num(r[ix["Warp Stall Sampling (All Samples)"]])
    if e < frac * tot_i and s < frac * tot_s:
        continue
    top = sorted(((num(r[h.index(k)]), k[6:]) for k in reasons), reverse=True)[:2]
    print(f"{r[ix['Address']]:>8} {100 * e / tot_i:5.2f}% {100 * s / tot_s:5.2f}%  {r[ix['Source']][:70]:70s} "
          + " ".join(f"{k}:{int(v)}" for v, k in top if v))
