"""Golden pass 2 alone on C2 (fi_golden_trace_jit_range over every warp), with
and without the fused profile, CUDA events, best of `reps`; the fused counts are
checked against K1 over the trace the pass wrote.
usage: golden_pass2_ab.py [reps]"""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from fi_inputs import programs as P  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
dp = fi.DeviceProgram(P.c2(full=True), "cuda:0")
jit = dp.jit(fi.FI_JIT_GOLDEN)
gt = fi.golden_run(dp)
st = fi.DeviceStatus(dp.device)
W = dp.n_warps
ic = torch.zeros((dp.n_inst, 8), dtype=torch.int64, device=dp.device)
cc = torch.zeros((gt.n_chunks, 8), dtype=torch.int32, device=dp.device)


def once(prof):
    if prof:
        ic.zero_()
        cc.zero_()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fi._check(fi.lib().fi_golden_trace_jit_range(jit.h, C.byref(dp.c), fi._p(gt.image), C.byref(gt.c), 0, W, 0, W,
                                                 fi._p(ic) if prof else None, fi._p(cc) if prof else None,
                                                 fi._p(st.t), fi._stream()), "fi_golden_trace_jit_range")
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b)


for prof in (False, True, False, True):
    print(f"pass 2, fused profile {'on ' if prof else 'off'}: {min(once(prof) for _ in range(reps)):.3f} ms", flush=True)
k1 = fi.profile(gt)
print("fused == K1:", bool(torch.equal(k1[0], ic)), bool(torch.equal(k1[1], cc)), flush=True)
