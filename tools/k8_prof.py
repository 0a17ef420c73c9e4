"""K8 (fi_classify_batched, JIT re-execution) on a full-size multi-launch
program, for ncu: golden run, profile, select n replicas, K4, then one timed
K8 call (CUDA events) and the outcome digest.
usage: k8_prof.py C3|C4|stencil|lbm|md|ep|cg [n] [batch] [mem_budget_GB]"""
import hashlib
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fi_inputs import hpc as H, programs as P, resnet as R  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 128
batch = int(sys.argv[3]) if len(sys.argv) > 3 and int(sys.argv[3]) > 0 else None
budget = int(sys.argv[4]) << 30 if len(sys.argv) > 4 else 24 << 30
if cfg == "C3":
    prog, seed = P.c3(full=True), P.CAMPAIGN_SEED[3]
elif cfg == "C4":
    prog, seed = R.c4(full=True), R.C4_CAMPAIGN_SEED
else:
    names = ["stencil", "lbm", "md", "ep", "cg"]
    prog, seed = H.c5(full=True)[names.index(cfg)], H.C5_CAMPAIGN_SEED + names.index(cfg)
torch.cuda.set_device(0)
dp = fi.DeviceProgram(prog)
t0 = time.time()
dp.jit(fi.FI_JIT_INJECT | fi.FI_JIT_GOLDEN | fi.FI_JIT_PAGE)
gt = fi.golden_run(dp)
ic, cc = fi.profile(gt)
sites = fi.select_sites(fi.SiteIndex(gt, ic, cc), fi.schedule(seed, [fi.G_GP], [0]), 0, n)
cap = fi.log_capacity(gt)
out, log = fi.inject(gt, sites, n, cap)
torch.cuda.synchronize()
print(f"setup {time.time() - t0:.1f} s, {dp.n_inst} launches, {gt.n_rec} records", flush=True)
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
hist = fi.classify_batched(gt, sites, n, out, log, cap, batch=batch, engine="jit", mem_budget=budget)
b.record()
torch.cuda.synchronize()
ms = a.elapsed_time(b)
dig = hashlib.sha1(out.cpu().numpy().tobytes()).hexdigest()[:16]
print(f"K8 {cfg} n={n}: {ms:.1f} ms = {n / (ms / 1e3):.1f} replicas/s, hist {hist.sum((0, 1)).tolist()}, "
      f"out-digest {dig}", flush=True)
