"""Golden-run timing (both passes, JIT or interpreter engine) on C2 outside bench.py.
usage: golden_time.py [C2|mini] [jit|interp] [reps]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
engine = sys.argv[2] if len(sys.argv) > 2 else "jit"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
dp = fi.DeviceProgram(P.c2(full=(cfg == "C2")), "cuda:0")
if engine == "jit":
    dp.jit(fi.FI_JIT_GOLDEN)
for r in range(reps):
    torch.cuda.synchronize()
    t = time.perf_counter()
    gt = fi.golden_run(dp, engine=engine)
    torch.cuda.synchronize()
    print(f"golden {cfg} {engine}: {1e3 * (time.perf_counter() - t):.1f} ms, {gt.n_rec} records", flush=True)
    del gt
