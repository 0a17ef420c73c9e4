"""fi_campaign end to end on C2 (bench.py's e2e call) at several checkpoint
intervals, interleaved, 4 warm calls each: wall seconds and the golden / inject
stage times.  Diagnostic.  usage: e2e_ckpt_ab.py [interval ...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

ivs = [int(x) for x in sys.argv[1:]] or [4096, 8192, 16384]
prog = P.c2(full=True)
host = {k: torch.from_numpy(np.ascontiguousarray(getattr(prog, k)).view(np.uint8).reshape(-1).copy()).pin_memory()
        for k in ("code", "kernels", "instances", "cbank", "buffers", "init_image")}
res = {iv: [] for iv in ivs}
fi.campaign(prog, P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], 10000, 0, 1, host=host, engine="jit")
for rep in range(4):
    for iv in ivs:
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = fi.campaign(prog, P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], 10000, 0, 1, host=host, engine="jit",
                        ckpt=iv)
        res[iv].append((time.perf_counter() - t0, r.ms["golden"], r.ms["inject"], tuple(r.hist.sum(axis=(0, 1)))))
for iv in ivs:
    print(f"interval {iv}: wall s {[round(x[0], 4) for x in res[iv]]} golden ms {[round(x[1], 1) for x in res[iv]]} "
          f"inject ms {[round(x[2], 2) for x in res[iv]]} outcomes {res[iv][0][3]}", flush=True)
