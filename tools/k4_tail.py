"""Where K4's tail comes from on C2: outcome / fault kind mix and the emulated
length of each replica class (golden remaining steps; watchdog replicas run to
10 L + 1024).  Diagnostic only."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 10000
prog = P.c2(full=True)
dp = fi.DeviceProgram(prog)
gt = fi.golden_run(dp)
ic, cc = fi.profile(gt)
idx = fi.SiteIndex(gt, ic, cc)
sites = fi.select_sites(idx, fi.schedule(P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3]), 0, n)
cap = fi.log_capacity(gt)
for _ in range(2):
    torch.cuda.synchronize(); t = time.time()
    out, log = fi.inject(gt, sites, n, cap)
    torch.cuda.synchronize(); print("inject s", time.time() - t)
inj = fi.as_numpy(out, fi.INJ_DTYPE, n)
st = fi.as_numpy(sites, fi.SITE_DTYPE, n)
L = gt.warp_len.cpu().numpy()[st["warp"]]
# restart step of each replica: the last golden checkpoint at or before its site
# (checkpoint c's step is stored in its last row, ~0 when absent; no checkpoints: 0)
start = np.zeros(n, dtype=np.int64)
if gt.ckpt is not None and gt.ckpt_interval:
    iv, rows = gt.ckpt_interval, gt.dp.n_regs + 4
    ck = gt.ckpt.cpu().numpy().view(np.uint32)
    off = gt.ckpt_off.cpu().numpy()
    for i in range(n):
        c = int(st["step"][i]) // iv
        while c > 0 and ck[(off[st["warp"][i]] + c) * rows * 32 + (rows - 1) * 32] > st["step"][i]:
            c -= 1
        start[i] = ck[(off[st["warp"][i]] + c) * rows * 32 + (rows - 1) * 32]
rem = L - start
for k in range(5):
    m = inj["fault_kind"] == k
    if m.any():
        print("fault_kind", k, "n", int(m.sum()), "golden remaining steps mean", float(rem[m].mean()),
              "max", int(rem[m].max()), "emulated est", float(np.where(k == 3, 10 * L[m] + 1024 - start[m], rem[m]).mean()))
tot = np.where(inj["fault_kind"] == 3, 10 * L + 1024 - start, rem)
print("total est emulated steps", int(tot.sum()), "of which watchdog", int(tot[inj["fault_kind"] == 3].sum()))
wd = inj["fault_kind"] == 3
print("watchdog sites: dst_reg", np.unique(st["dst_reg"][wd], return_counts=True), "pc", np.unique(st["pc"][wd], return_counts=True))

# solo latency of individual replicas: time / golden-remaining steps exposes
# replicas whose faulty continuation leaves the emulator's fast paths
rng = np.random.default_rng(1)
pick = rng.choice(n, 300, replace=False)
res = []
for i in pick:
    sub = sites[i * 64:(i + 1) * 64]
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    o, lg = fi.inject(gt, sub, 1, cap)
    e1.record(); torch.cuda.synchronize()
    res.append((e0.elapsed_time(e1), int(rem[i]), i))
res.sort(key=lambda r: -r[0] / max(r[1], 1))
rate = np.median([r[1] / r[0] for r in res if r[1] > 10000])
print("median solo steps/ms", rate)
for ms, rm, i in res[:15]:
    print(f"ms {ms:.2f} rem {rm} steps/ms {rm / ms:.0f} pc {st['pc'][i]} dst {st['dst_reg'][i]} bfm {st['bfm'][i]} "
          f"lane {st['lane'][i]} fk {inj['fault_kind'][i]} out {inj['outcome'][i]} mask {st['mask'][i]:#x}")
print("slowest absolute:", sorted(res, key=lambda r: -r[0])[:5])
