"""The G-rank split of C2's replica set, measured on one GPU: each rank's share
(select + K4 + K5 of its replicas) timed alone, for the contiguous replica blocks
[r*n/G, (r+1)*n/G) and for the cost-balanced split (replicas in longest-first order
by their estimated emulated steps, dealt to the ranks in snake order).
usage: shard_split.py [G] [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign  # noqa: E402

G = int(sys.argv[1]) if len(sys.argv) > 1 else 8
n = int(sys.argv[2]) if len(sys.argv) > 2 else 10000
camp = Campaign(P.c2(full=True), P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], n, 0, 1, "cuda:0", engine="jit")
camp.step()
torch.cuda.synchronize()
sites = camp.sites_np().copy()
gt = camp.gt
L = gt.warp_len.cpu().numpy()[sites["warp"]].astype(np.int64)
iv = gt.ckpt_interval
start = (sites["step"].astype(np.int64) // iv) * iv if iv else np.zeros(n, np.int64)
est = L - start


def run(idx, reps=3):
    sub = torch.from_numpy(sites[idx].view(np.uint8).copy()).to(camp.device)
    m = len(idx)
    best = None
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fi.inject(gt, sub, m, camp.cap, camp.out, camp.log, camp.status, camp.inj_ws, engine="jit")
        h = torch.zeros((8, 4, 3), dtype=torch.int64, device=camp.device)
        fi.classify(gt, sub, m, camp.out, camp.log, camp.cap, h, camp.status)
        b.record()
        torch.cuda.synchronize()
        best = a.elapsed_time(b) if best is None else min(best, a.elapsed_time(b))
    return best


full = run(np.arange(n))
blocks = [run(np.arange(r * n // G, (r + 1) * n // G)) for r in range(G)]
order = np.argsort(-est, kind="stable")
rnd, pos = np.arange(n) // G, np.arange(n) % G
rank_of = np.where(rnd % 2 == 0, pos, G - 1 - pos)
balanced = [run(np.sort(order[rank_of == r])) for r in range(G)]
print(f"full {full:.3f} ms")
print(f"contiguous blocks: {[round(x, 3) for x in blocks]} slowest {max(blocks):.3f} ratio {full / max(blocks):.2f} "
      f"(est steps per rank {[int(est[r * n // G:(r + 1) * n // G].sum()) for r in range(G)]})")
print(f"balanced (LPT snake): {[round(x, 3) for x in balanced]} slowest {max(balanced):.3f} ratio {full / max(balanced):.2f} "
      f"(est steps per rank {[int(est[order[rank_of == r]].sum()) for r in range(G)]})")
