"""Small driver for ncu captures: C2 golden run, one profile, index, select,
inject, classify (n replicas).  Never a bench number (runs under ncu)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 2048
prog = P.c2(full=(cfg == "C2"))
dp = fi.DeviceProgram(prog)
gt = fi.golden_run(dp)
ic, cc = fi.profile(gt)
idx = fi.SiteIndex(gt, ic, cc)
sites = fi.select_sites(idx, fi.schedule(P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3]), 0, n)
cap = fi.log_capacity(gt)
out, log = fi.inject(gt, sites, n, cap)
hist = fi.classify(gt, sites, n, out, log, cap)
torch.cuda.synchronize()
print("hist", hist.sum(dim=(0, 1)).tolist())
