"""K4 latency of single replicas (the bound on the injection stage when a GPU
holds fewer replicas than it has resident warps — the G = 8 shard of C2):
C2 campaign step, then K4 on sub-sets of the replica set, CUDA events.
usage: k4_latency.py [n_longest]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign  # noqa: E402

k = int(sys.argv[1]) if len(sys.argv) > 1 else 4
camp = Campaign(P.c2(full=True), P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], 10000, 0, 1, "cuda:0", engine="jit")
camp.step()
torch.cuda.synchronize()
sites = camp.sites_np().copy()
inj = camp.inj_np().copy()
gt = camp.gt
L = gt.warp_len.cpu().numpy()[sites["warp"]].astype(np.int64)
iv = gt.ckpt_interval
start = (sites["step"].astype(np.int64) // iv) * iv if iv else np.zeros(len(sites), np.int64)
est = np.where(inj["fault_kind"] == 3, 10 * L + 1024, L) - start       # emulated steps estimate


def run(idx, reps=3):
    sub = torch.from_numpy(sites[idx].view(np.uint8).copy()).to(camp.device)
    n = len(idx)
    best = None
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fi.inject(gt, sub, n, camp.cap, camp.out, camp.log, camp.status, camp.inj_ws, engine="jit")
        b.record()
        torch.cuda.synchronize()
        best = a.elapsed_time(b) if best is None else min(best, a.elapsed_time(b))
    steps = int(camp.inj_ws[8:16].cpu().view(torch.int64).item())
    return best, steps


order = np.argsort(-est)
print("fault kinds:", np.bincount(inj["fault_kind"], minlength=5).tolist(), "est steps max", int(est.max()),
      "median", int(np.median(est)))
for i in order[:k]:
    ms, steps = run(np.array([i]))
    print(f"replica {i}: fault_kind {inj['fault_kind'][i]} est {est[i]} emulated {steps} steps in {ms:.3f} ms "
          f"= {steps / ms / 1e3:.1f} steps/us alone", flush=True)
for m in (148, 1250, 10000):
    idx = order[:m]
    ms, steps = run(idx)
    print(f"longest {m}: {ms:.3f} ms, {steps} steps, {steps / ms / 1e3:.1f} steps/us", flush=True)
ms, steps = run(np.arange(1250))
print(f"block [0,1250): {ms:.3f} ms, {steps} steps", flush=True)
