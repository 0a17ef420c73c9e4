"""Is K4's tail a few long replicas?  Time all replicas, then without the slowest
solo ones.  Diagnostic only."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

n = 10000
prog = P.c2(full=True)
dp = fi.DeviceProgram(prog)
gt = fi.golden_run(dp)
ic, cc = fi.profile(gt)
idx = fi.SiteIndex(gt, ic, cc)
sites = fi.select_sites(idx, fi.schedule(P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3]), 0, n)
cap = fi.log_capacity(gt)
st = fi.as_numpy(sites, fi.SITE_DTYPE, n)


def timed(sub, m, reps=3):
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fi.inject(gt, sub, m, cap)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


print("all", timed(sites, n))
# solo time of every KCNT-site replica (loop counter corruptions diverge)
kc = np.nonzero(st["dst_reg"] == P.KCNT)[0]
solo = []
for i in kc:
    solo.append((timed(sites[i * 64:(i + 1) * 64], 1, 1), int(i)))
solo.sort(reverse=True)
print("KCNT replicas", len(kc), "top solo ms", solo[:8])
keep = np.setdiff1d(np.arange(n), [i for _, i in solo[:4]])
sub = sites.view(-1, 64)[torch.from_numpy(keep).cuda()].reshape(-1)
print("without top-4 KCNT", timed(sub, len(keep)))
keep = np.setdiff1d(np.arange(n), kc)
sub = sites.view(-1, 64)[torch.from_numpy(keep).cuda()].reshape(-1)
print("without all KCNT", timed(sub, len(keep)), len(keep))
