"""Checkpoint interval trade-off on C2 (diagnostic): golden run time (the trace
pass runs in step mode around every checkpoint) against K4 time (a replica
restarts from the checkpoint at or before its site).  Outputs must not depend on
the interval (digest).  usage: ck_sweep.py [C2|mini] [interval ...]"""
import hashlib
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
ivs = [int(x) for x in sys.argv[2:]] or [4096, 8192, 16384]
n = 10000
camp = Campaign(P.c2(full=(cfg == "C2")), P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], n, 0, 1, "cuda:0", engine="jit")
for iv in ivs:
    camp.gt = None
    torch.cuda.empty_cache()
    gms = []
    for _ in range(2):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        gt = fi.golden_run(camp.dp, iv, engine="jit")
        torch.cuda.synchronize()
        gms.append((time.perf_counter() - t0) * 1e3)
        if _ == 0:
            del gt
    camp.gt = gt
    camp.step()
    torch.cuda.synchronize()
    ms = []
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fi.inject(camp.gt, camp.sites, n, camp.cap, camp.out, camp.log, camp.status, camp.inj_ws, engine="jit")
        b.record()
        torch.cuda.synchronize()
        ms.append(a.elapsed_time(b))
    steps = int(camp.inj_ws[8:16].cpu().view(torch.int64).item())
    camp.check()
    dig = hashlib.sha1(camp.out.cpu().numpy().tobytes()).hexdigest()[:16]
    print(f"interval {iv}: golden ms {[round(x, 1) for x in gms]} K4 best {min(ms):.2f} ms steps {steps} "
          f"out-digest {dig}", flush=True)
