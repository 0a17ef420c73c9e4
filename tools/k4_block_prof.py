"""K4 on one rank's replica block alone vs its longest replica alone (C2), for
ncu: the campaign step (one K4 launch), then K4 on replicas [0, n/G) and K4 on
the block's longest replica.  Capture the last two launches with
ncu -k regex:k_inject_jit --launch-skip 1 -c 2.
usage: k4_block_prof.py [G]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign  # noqa: E402

G = int(sys.argv[1]) if len(sys.argv) > 1 else 8
camp = Campaign(P.c2(full=True), P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], 10000, 0, 1, "cuda:0", engine="jit")
camp.step()
torch.cuda.synchronize()
sites = camp.sites_np().copy()
gt = camp.gt
m = len(sites) // G
L = gt.warp_len.cpu().numpy()[sites["warp"][:m]].astype(np.int64)
iv = gt.ckpt_interval
start = (sites["step"][:m].astype(np.int64) // iv) * iv if iv else np.zeros(m, np.int64)
longest = int(np.argmax(L - start))


def run(idx):
    sub = torch.from_numpy(sites[idx].view(np.uint8).copy()).to(camp.device)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fi.inject(gt, sub, len(idx), camp.cap, camp.out, camp.log, camp.status, camp.inj_ws, engine="jit")
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b), int(camp.inj_ws[8:16].cpu().view(torch.int64).item())


ms, steps = run(np.arange(m))
print(f"block [0,{m}): {ms:.3f} ms, {steps} steps", flush=True)
ms, steps = run(np.array([longest]))
print(f"its longest replica {longest}: {ms:.3f} ms, {steps} steps", flush=True)
