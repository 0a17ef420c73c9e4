"""One C2 replica alone on the GPU (the longest one: its site in the first
checkpoint interval of its warp), for ncu: the campaign step (one K4 launch), then
K4 on that replica three times (the last ones find its lines in L2).  Capture the
third with ncu -k regex:k_inject_jit --launch-skip 3 -c 1.
usage: k4_lone.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign  # noqa: E402

camp = Campaign(P.c2(full=True), P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], 10000, 0, 1, "cuda:0", engine="jit")
camp.step()
torch.cuda.synchronize()
sites = camp.sites_np().copy()
gt = camp.gt
L = gt.warp_len.cpu().numpy()[sites["warp"]].astype(np.int64)
iv = gt.ckpt_interval
start = (sites["step"].astype(np.int64) // iv) * iv if iv else np.zeros(len(sites), np.int64)
i = int(np.argmax(L - start))
sub = torch.from_numpy(sites[[i]].view(np.uint8).copy()).to(camp.device)
for r in range(3):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fi.inject(gt, sub, 1, camp.cap, camp.out, camp.log, camp.status, camp.inj_ws, engine="jit")
    b.record()
    torch.cuda.synchronize()
    steps = int(camp.inj_ws[8:16].cpu().view(torch.int64).item())
    print(f"replica {i} alone: {a.elapsed_time(b):.3f} ms, {steps} steps", flush=True)
