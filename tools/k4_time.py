"""K4 (fi_inject_jit) timing on the bench's replica set, outside bench.py:
C2 golden run + one profile/index/select, then R timed K4 launches (CUDA
events) and the outputs' digest (to compare variants bit-for-bit).
usage: k4_time.py [C2|mini] [replicas] [reps]    (env FI_JIT_MIN_BLOCKS etc.)"""
import hashlib
import numpy as np
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 10000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
prog = P.c2(full=(cfg == "C2"))
t0 = time.time()
camp = Campaign(prog, P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], n, 0, 1, "cuda:0", engine="jit")
camp.step()
torch.cuda.synchronize()
print(f"setup {time.time() - t0:.1f} s", flush=True)
ms = []
for _ in range(reps):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fi.inject(camp.gt, camp.sites, n, camp.cap, camp.out, camp.log, camp.status, camp.inj_ws, engine="jit")
    b.record()
    torch.cuda.synchronize()
    ms.append(a.elapsed_time(b))
steps = int(camp.inj_ws[8:16].cpu().view(torch.int64).item())
camp.check()
dig = hashlib.sha1(camp.out.cpu().numpy().tobytes()).hexdigest()[:16]
print(f"K4 {cfg} n={n}: ms {sorted(ms)} best {min(ms):.2f} steps {steps} "
      f"rate {steps / (min(ms) / 1e3):.3e} warp-inst/s out-digest {dig} "
      f"min_blocks={os.environ.get('FI_JIT_MIN_BLOCKS', '3')}", flush=True)
if os.environ.get("K4_SUBSETS"):
    # where the K4 tail comes from: time the replicas that ended in a fault/watchdog
    # (fault_kind != 0) apart from the rest
    inj = fi.as_numpy(camp.out, fi.INJ_DTYPE, n)
    st = camp.sites.view(-1, 64)
    for name, mask in (("no-fault", inj["fault_kind"] == 0), ("fault", inj["fault_kind"] != 0)):
        idx = torch.from_numpy(np.nonzero(mask)[0]).to(st.device)
        m = int(idx.numel())
        sub = st[idx].contiguous().view(-1)
        out2 = torch.empty(m * 24, dtype=torch.uint8, device=st.device)
        log2 = torch.empty(m * camp.cap * 16, dtype=torch.uint8, device=st.device)
        ws2 = torch.empty(fi.lib().fi_inject_workspace(m), dtype=torch.uint8, device=st.device)
        best = 1e9
        for _ in range(3):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fi.inject(camp.gt, sub, m, camp.cap, out2, log2, camp.status, ws2, engine="jit")
            b.record()
            torch.cuda.synchronize()
            best = min(best, a.elapsed_time(b))
        s2 = int(ws2[8:16].cpu().view(torch.int64).item())
        print(f"subset {name}: {m} replicas, {best:.2f} ms, {s2} steps ({s2 / max(m, 1):.0f}/replica), "
              f"fault kinds {np.bincount(inj['fault_kind'][mask], minlength=5).tolist()}", flush=True)
