"""Secondary measurements on the multi-launch configs (C3, C4, C5 programs):
golden run, exact profile (K1, HBM rate), index + select, K4, K8 outcomes for a
bounded replica sample.  One JSON line per program.  Not the bench contract's
line (bench.py measures C2); the numbers go to profiles/ and DESIGN.md.

usage: secondary_bench.py C3|C4|C5 [replicas] [batch]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from fi_inputs import hpc as H, programs as P, resnet as R  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402


def timed(f, reps=1):
    best = None
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        r = f()
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        best = ms if best is None else min(best, ms)
    return r, best


ENGINE = os.environ.get("FI_ENGINE", "jit")        # jit | interp


def run(name, prog, seed, n, batch):
    dp = fi.DeviceProgram(prog)
    jit_s = 0.0
    if ENGINE == "jit":                               # one module: golden passes, K4, K8 (setup, reported)
        t0 = time.time()
        dp.jit(fi.FI_JIT_INJECT | fi.FI_JIT_GOLDEN | fi.FI_JIT_PAGE)
        jit_s = time.time() - t0
    t0 = time.time()
    gt = fi.golden_run(dp, engine=ENGINE)
    torch.cuda.synchronize()
    golden_s = time.time() - t0
    (ic, cc), prof_ms = timed(lambda: fi.profile(gt), reps=3)
    counts = ic.cpu().numpy()
    counted = int(counts[:, 4].sum() + counts[:, 6].sum())
    nch = (gt.n_rec + 1023) // 1024
    algo = 16 * gt.n_rec + 32 * nch + 64 * dp.n_inst
    idx, idx_ms = timed(lambda: fi.SiteIndex(gt, ic, cc))
    sites, sel_ms = timed(lambda: fi.select_sites(idx, fi.schedule(seed, [fi.G_GP], [0]), 0, n))
    cap = fi.log_capacity(gt)
    (out, log), k4_ms = timed(lambda: fi.inject(gt, sites, n, cap, engine=ENGINE))
    hist, k8_ms = timed(lambda: fi.classify_batched(gt, sites, n, out, log, cap, batch=batch, engine=ENGINE))
    inj = fi.as_numpy(out, fi.INJ_DTYPE, n)
    oc = np.bincount(np.minimum(inj["outcome"], 4), minlength=5)
    line = {"program": name, "instances": dp.n_inst, "static_kernels": len(prog.kernels), "warps": dp.n_warps,
            "records": gt.n_rec, "counted_thread_instrs": counted, "golden_s": golden_s,
            "profile_ms": prof_ms, "profile_thread_instrs_per_s": counted / (prof_ms / 1e3),
            "profile_hbm_gbs": algo / (prof_ms / 1e3) / 1e9, "index_ms": idx_ms, "select_ms": sel_ms,
            "replicas": n, "k4_ms": k4_ms, "k8_ms": k8_ms,
            "injections_per_s": n / ((sel_ms + k4_ms + k8_ms) / 1e3),
            "outcomes": {"masked": int(oc[0]), "sdc": int(oc[1]), "due": int(oc[2]),
                         "unclassified_wild_load": int(((inj["outcome"] == 0xFF) & (inj["flags"] & 4 > 0)).sum()),
                         "unclassified_capacity": int(((inj["outcome"] == 0xFF) & (inj["flags"] & 2 > 0)).sum())},
            "group": "G_GP", "bfm": "FLIP_SINGLE_BIT", "engine": ENGINE, "jit_compile_s": jit_s}
    print(json.dumps(line), flush=True)
    del gt, dp
    torch.cuda.empty_cache()


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 200
    batch = int(sys.argv[3]) if len(sys.argv) > 3 else None          # None: sized to the memory budget
    if cfg == "C3":
        run("C3 CG 512x256, 500 iterations", P.c3(full=True), P.CAMPAIGN_SEED[3], n, batch)
    elif cfg == "C4":
        run("C4 ResNet-50 v1.5, 224x224, batch 1", R.c4(full=True), R.C4_CAMPAIGN_SEED, n, batch)
    elif cfg == "C5":
        for i, prog in enumerate(H.c5(full=True)):
            run("C5 " + prog.meta["config"], prog, H.C5_CAMPAIGN_SEED + i, n, batch)


if __name__ == "__main__":
    main()
