"""Full-size C3 probe: golden run, exact + approximate profile, index, select (timed)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

t = time.time()
prog = P.c3(full=True)
print("gen", time.time() - t, len(prog.instances), prog.n_warps, prog.image_bytes / 1e9, "GB", flush=True)
t = time.time()
dp = fi.DeviceProgram(prog)
gt = fi.golden_run(dp)
torch.cuda.synchronize()
print("golden", time.time() - t, "records", gt.n_rec, flush=True)
ev = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
for rep in range(3):
    ev[0].record()
    ic, cc = fi.profile(gt)
    ev[1].record()
    idx = fi.SiteIndex(gt, ic, cc)
    ev[2].record()
    sites = fi.select_sites(idx, fi.schedule(P.CAMPAIGN_SEED[3], [fi.G_GP], [0]), 0, 10000)
    ev[3].record()
    ap = fi.profile_approx(gt)
    ev[4].record()
    torch.cuda.synchronize()
    print("profile ms", ev[0].elapsed_time(ev[1]), "index", ev[1].elapsed_time(ev[2]), "select",
          ev[2].elapsed_time(ev[3]), "approx", ev[3].elapsed_time(ev[4]), flush=True)
c = ic.cpu().numpy()
counted = int(c[:, 4].sum() + c[:, 6].sum())
print("counted", counted, "thread-instrs/s", counted / (ev[0].elapsed_time(ev[1]) / 1e3))
print("approx==exact", bool((ap.cpu().numpy() == c).all()))
s = fi.as_numpy(sites, fi.SITE_DTYPE, 10000)
print("sites instances", np.bincount(prog.instances["kernel"][s["instance"]], minlength=12))
