"""fi_campaign on C2 called repeatedly from pinned host buffers (bench.py's e2e
leg): wall time, the call's own stage times and the device's free memory after
each call.  usage: e2e_repeat.py [calls]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

calls = int(sys.argv[1]) if len(sys.argv) > 1 else 6
prog = P.c2(full=True)
host = {k: torch.from_numpy(np.ascontiguousarray(getattr(prog, k)).view(np.uint8).reshape(-1).copy()).pin_memory()
        for k in ("code", "kernels", "instances", "cbank", "buffers", "init_image")}
torch.cuda.set_device(0)
for it in range(calls):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = fi.campaign(prog, P.CAMPAIGN_SEED[2], [fi.G_GP], [0, 1, 2, 3], 10000, host=host, engine="jit")
    dt = time.perf_counter() - t0
    free, total = torch.cuda.mem_get_info()
    print(f"call {it}: {dt * 1e3:.1f} ms, free {free / 2**30:.1f} GiB, stages "
          + " ".join(f"{k} {v:.2f}" for k, v in r.ms.items()), flush=True)
