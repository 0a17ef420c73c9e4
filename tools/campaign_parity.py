"""Full-size multi-launch campaigns (BASELINE configs[2..4]: C3, C4, C5) on one
B200, with oracle parity on a stratified subset.  One JSON line per program to
stdout (and appended to --out):

  GPU   golden run (JIT), K1 profile, index, K3 select of ALL n replicas, K4,
        K8 whole-program outcomes (JIT re-execution) — CUDA-event times,
        injections/s = n / (select + K4 + K8);
  oracle (CPU, the definition: PAPER.md:72 step (4), :206) — its own golden run
        with the trace kept, its own selection of ALL n replicas (every site
        field compared with the GPU's), and FULL-mode injection (the whole
        program re-run with the corruption, outputs compared bitwise) of the
        replicas j = k * (n // subset); outcome, flags and fault kind compared.

usage: campaign_parity.py C3|C4|C5 [--n N] [--subset S] [--programs i,j] [--out F]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle as O  # noqa: E402
from fi_inputs import hpc as H, programs as P, resnet as R  # noqa: E402
from paper_conf_dsn_0002hsvk21_b200 import fi  # noqa: E402


def ev_time(f):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    r = f()
    e1.record()
    torch.cuda.synchronize()
    return r, e0.elapsed_time(e1)


def run(name, prog, seed, groups, bfms, n, subset, out_path):
    line = {"program": name, "instances": len(prog.instances), "warps": prog.n_warps, "replicas": n,
            "groups": [O.GROUP_NAMES[g] for g in groups], "bfms": bfms}
    t0 = time.time()
    dp = fi.DeviceProgram(prog)
    dp.jit(fi.FI_JIT_INJECT | fi.FI_JIT_GOLDEN | fi.FI_JIT_PAGE)
    line["jit_compile_s"] = time.time() - t0
    t0 = time.time()
    gt = fi.golden_run(dp)
    torch.cuda.synchronize()
    line["golden_s"] = time.time() - t0
    line["records"] = gt.n_rec
    (ic, cc), line["profile_ms"] = ev_time(lambda: fi.profile(gt))
    counts = ic.cpu().numpy()
    line["profile_thread_instrs_per_s"] = int(counts[:, 4].sum() + counts[:, 6].sum()) / (line["profile_ms"] / 1e3)
    sched = fi.schedule(seed, groups, bfms)
    idx, line["index_ms"] = ev_time(lambda: fi.SiteIndex(gt, ic, cc))
    sites, line["select_ms"] = ev_time(lambda: fi.select_sites(idx, sched, 0, n))
    cap = fi.log_capacity(gt)
    (out, log), line["k4_ms"] = ev_time(lambda: fi.inject(gt, sites, n, cap, engine="jit"))
    hist, line["k8_ms"] = ev_time(lambda: fi.classify_batched(gt, sites, n, out, log, cap, engine="jit"))
    line["injections_per_s"] = n / ((line["select_ms"] + line["k4_ms"] + line["k8_ms"]) / 1e3)
    gs = fi.as_numpy(sites, fi.SITE_DTYPE, n).copy()
    gi = fi.as_numpy(out, fi.INJ_DTYPE, n).copy()
    h = hist.cpu().numpy()
    line["outcomes"] = {"masked": int(h[..., 0].sum()), "sdc": int(h[..., 1].sum()), "due": int(h[..., 2].sum()),
                        "unclassified": int((gi["outcome"] == 0xFF).sum())}
    del gt, dp, out, log, sites, idx, hist
    torch.cuda.empty_cache()

    # ---- the oracle: its own golden run, selection of every replica, full-mode subset
    t0 = time.time()
    g = O.Golden(prog)
    assert (g.counts() == counts.astype(np.uint64)).all(), "profile counts differ from the oracle"
    osites = g.select(seed, groups, bfms, 0, n)
    line["oracle_golden_select_s"] = time.time() - t0
    bad_site = [f for f in osites.dtype.names if not (osites[f] == gs[f]).all()]
    js = np.arange(0, n, max(1, n // subset))[:subset]
    t0 = time.time()
    oi = g.inject(osites[js], O.MODE_FULL)
    line["oracle_full_s"] = time.time() - t0
    line["oracle_cores"] = O.n_threads_default()
    mism = {f: int((oi[f] != gi[js][f]).sum()) for f in ("outcome", "flags", "fault_kind")}
    line["parity"] = {"sites_all_n": "identical" if not bad_site else f"DIFFER in {bad_site}",
                      "counts": "identical", "subset": len(js), "subset_rule": f"j = k * {max(1, n // subset)}",
                      "outcome_flags_fault_kind": "identical" if not any(mism.values()) else mism,
                      "subset_outcomes": np.bincount(oi["outcome"], minlength=3).tolist()}
    print(json.dumps(line), flush=True)
    if out_path:
        with open(out_path, "a") as f:
            f.write(json.dumps(line) + "\n")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", choices=["C3", "C4", "C5"])
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--subset", type=int, default=None)
    ap.add_argument("--programs", default=None, help="C5: comma-separated program indices")
    ap.add_argument("--n-list", default=None, help="C5: comma-separated replica counts, one per selected program")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    if a.config == "C3":
        run("C3 CG 512x256, 500 iterations (5,002 launches)", P.c3(full=True), P.CAMPAIGN_SEED[3], [fi.G_GP], [0],
            a.n or 10000, a.subset or 64, a.out)
    elif a.config == "C4":
        run("C4 ResNet-50 v1.5 224x224 batch 1 (72 launches)", R.c4(full=True), R.C4_CAMPAIGN_SEED, [fi.G_GP], [0],
            a.n or 100000, a.subset or 32, a.out)
    else:
        progs = H.c5(full=True)
        sel = list(range(len(progs))) if a.programs is None else [int(x) for x in a.programs.split(",")]
        ns = [int(x) for x in a.n_list.split(",")] if a.n_list else [a.n or 2000] * len(sel)
        for i, n in zip(sel, ns):
            run("C5 " + progs[i].meta["config"], progs[i], H.C5_CAMPAIGN_SEED + i, [fi.G_GP], [0],
                n, a.subset or 16, a.out)


if __name__ == "__main__":
    main()
