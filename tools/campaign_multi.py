"""Full-size multi-launch campaign with K8 outcomes: C3 (5,002 launches), or C4
(env C4=1: ResNet-50 shape, 72 launches); env C3_MINI=1 for the mini sizes.
Golden run, exact profile, index, select n replicas, K4, K8; prints stage
times and outcomes.
Optionally checks a sample of replicas against the oracle's full mode."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P, resnet as R  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 200
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 512
n_oracle = int(sys.argv[3]) if len(sys.argv) > 3 else 0
full = os.environ.get("C3_MINI") is None
prog = (R.c4(full=full) if os.environ.get("C4") else P.c3(full=full))
t0 = time.time()
dp = fi.DeviceProgram(prog)
gt = fi.golden_run(dp)
torch.cuda.synchronize()
print("golden s", time.time() - t0, "records", gt.n_rec, "instances", dp.n_inst, flush=True)


def timed(f):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    r = f()
    e1.record()
    torch.cuda.synchronize()
    return r, e0.elapsed_time(e1)


(ic, cc), ms = timed(lambda: fi.profile(gt))
print("profile ms", ms, flush=True)
idx, ms = timed(lambda: fi.SiteIndex(gt, ic, cc))
print("index ms", ms)
sched = fi.schedule((R.C4_CAMPAIGN_SEED if os.environ.get("C4") else P.CAMPAIGN_SEED[3]), [fi.G_GP], [0])
sites, ms = timed(lambda: fi.select_sites(idx, sched, 0, n))
print("select ms", ms)
cap = fi.log_capacity(gt)
(out, log), ms = timed(lambda: fi.inject(gt, sites, n, cap))
print("K4 ms", ms, flush=True)
hist, ms = timed(lambda: fi.classify_batched(gt, sites, n, out, log, cap, batch=batch))
inj = fi.as_numpy(out, fi.INJ_DTYPE, n)
print("K8 ms", ms, "outcomes", np.bincount(inj["outcome"], minlength=4).tolist(),
      "injections/s", n / (ms / 1e3), flush=True)
if n_oracle:
    import oracle as O
    t1 = time.time()
    g = O.Golden(prog)
    os_ = g.select((R.C4_CAMPAIGN_SEED if os.environ.get("C4") else P.CAMPAIGN_SEED[3]), [fi.G_GP], [0], 0, n_oracle)
    oi = g.inject(os_, O.MODE_FULL)
    same = (oi["outcome"] == inj["outcome"][:n_oracle]).all() and (oi["flags"] == inj["flags"][:n_oracle]).all()
    print("oracle full mode on", n_oracle, "replicas:", "identical" if same else "DIFFERENT",
          np.bincount(oi["outcome"], minlength=4).tolist(), "oracle s", time.time() - t1)
