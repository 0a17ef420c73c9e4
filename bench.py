#!/usr/bin/env python
"""Benchmark of the NVBitFI hot path on B200 (BASELINE.json metric):
thread-dyn-instrs profiled/sec and injections/sec (% HBM roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2|C1|mini]
                    [--replicas 10000] [--impl fi|reference]

Workload (config C2 = BASELINE.json configs[1]): the SGEMM-shaped 4096^3 trace
(8,192 warps, 2.45e9 records, 39 GB resident in HBM) — full 8-group profile +
10,000 injections across the four fault models (G_GP, bfm = j mod 4).

One step = the whole hot path over the resident trace: K1 profile (sharded by
record range at N > 1, counts all-reduced), K2 site index, K3 select, K4 inject,
K5 classify, histogram all-reduce.  The golden run that makes the trace
resident is setup (it is timed separately as part of `e2e`).

value     = thread-dyn-instrs profiled / s   (sum of counted thread-instrs over
            the K1 profile-stage time, max over ranks)
injections_per_s = replicas / (select + inject + classify time, max over ranks)
Timing: CUDA events on the launching stream, L2 flushed (256 MiB write) before
every timed step, barrier + synchronize on both sides, max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

STAGES = ["profile", "exchange", "index", "select", "inject", "classify", "end"]


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2", choices=["C1", "C2", "mini"])
    ap.add_argument("--replicas", type=int, default=None)
    ap.add_argument("--impl", default="fi", choices=["fi", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-secondary", action="store_true",
                    help="skip the C4 (ResNet-50-shaped, 72 launches) multi-launch campaign sample")
    return ap.parse_args()


def make_program(cfg):
    from fi_inputs import programs as P
    if cfg == "C1":
        return P.c1(), P.CAMPAIGN_SEED[1], [7], [0], 100
    if cfg == "mini":
        return P.c2(full=False), P.CAMPAIGN_SEED[2], [7], [0, 1, 2, 3], 10000
    return P.c2(full=True), P.CAMPAIGN_SEED[2], [7], [0, 1, 2, 3], 10000


def workload_name(cfg, n):
    return {"C1": f"C1 vector-add n=1024 trace, {n} single-bit injections",
            "mini": f"mini-C2 SGEMM 256^3 trace, {n} injections x 4 fault models",
            "C2": f"C2 SGEMM 4096^3 trace (8,192 warps, 2.45e9 records): full 8-group profile + {n} injections "
                  f"across 4 fault models"}[cfg]


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.samples = []
        self.all = []
        self.proc = None

    def start(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,power.draw")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                          "-i", str(self.idx), "-lms", "25"], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
        except FileNotFoundError:
            self.proc = None
            return
        self.th = threading.Thread(target=self._read, daemon=True)
        self.th.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 7:
                self.all.append((time.perf_counter(), parts))

    def window(self, t0, t1):
        """Keep the samples taken inside [t0, t1] (the timed region); if nvidia-smi
        produced none there (a very short region), the nearest one after t0."""
        inside = [p for t, p in self.all if t0 <= t <= t1]
        if not inside:
            after = [p for t, p in self.all if t >= t0]
            inside = after[:1]
        self.samples = inside

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[2 + i].lower() == "active"})
        loaded = [x for x in sm if x > 0.5 * (max(mx) if mx else 1)] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


ORACLE_WARPS = 1024          # cpu_baseline and --impl reference interpret the same warps [0, 1024)
ORACLE_SCAN_RECORDS = 1 << 27   # the trace-scan leg: the first 2^27 records (2 GiB) of the resident trace


def oracle_count_sample(prog):
    """The oracle's interpretive profile of a fixed bounded sample: warps
    [0, ORACLE_WARPS) of the workload (golden interpretation + Table II count)."""
    import oracle as O
    nt = O.n_threads_default()
    nw = min(prog.n_warps, ORACLE_WARPS)
    t = time.perf_counter()
    n_rec, c = O.count_warps(prog, 0, nw, nt)
    dt = time.perf_counter() - t
    return int(c[4] + c[6]), int(n_rec), dt, nw, nt


def cpu_baseline(prog, sites_np, camp=None, n_inj=1024):
    """The oracle as it stands, on this host's cores, over bounded samples of the
    same workload:
      value       interpretive count of warps [0, ORACLE_WARPS) (the same sample the
                  reference arm times each step);
      trace_scan  the profiler's count over the first ORACLE_SCAN_RECORDS records of
                  the resident trace, copied to host RAM first (copy not timed) —
                  the CPU counterpart of K1;
      injections  warp-local injection of replicas [0, n_inj)."""
    import oracle as O
    counted, n_rec, dt, nw, nt = oracle_count_sample(prog)
    out = {
        "value": counted / dt, "unit": "thread-dyn-instrs/s", "cores": nt, "kind": "oracle",
        "value_per_core": counted / dt / nt,
        "sample": f"oracle golden interpretation + Table II group count of warps [0,{nw}) of the workload "
                  f"({n_rec} warp-records, {counted} thread-instrs) in {dt:.2f}s",
    }
    if camp is not None:
        nr = min(camp.gt.n_rec, ORACLE_SCAN_RECORDS)
        host = camp.gt.rec[:16 * nr].cpu().numpy()
        reps, t = 0, time.perf_counter()
        while True:                                # repeat the scan for >= 2 s of CPU work
            c = O.scan_trace(host, camp.dp.n_inst, nt)
            reps += 1
            ds = time.perf_counter() - t
            if ds >= 2.0:
                break
        ds /= reps
        cs = int(c[:, 4].sum() + c[:, 6].sum())
        out["trace_scan"] = {"value": cs / ds, "unit": "thread-dyn-instrs/s", "cores": nt,
                             "value_per_core": cs / ds / nt, "records_per_s": nr / ds, "gb_per_s": 16 * nr / ds / 1e9,
                             "sample": f"oracle scan (orc_scan_trace) of records [0,{nr}) of the resident trace "
                                       f"({16 * nr / 2**30:.1f} GiB in host RAM, D2H not timed): {ds:.3f}s per scan, mean of {reps}"}
        del host
    ni = min(len(sites_np), n_inj)
    t = time.perf_counter()
    O.inject_local(prog, sites_np[:ni], nt)
    di = time.perf_counter() - t
    out["injections_per_s"] = ni / di
    out["injections_per_s_per_core"] = ni / di / nt
    out["injection_sample"] = (f"oracle warp-local injection (golden + faulty re-execution of the site's warp, "
                               f"classification) of replicas [0,{ni}) in {di:.2f}s")
    return out


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle as the reference arm (rank 0 only)."""
    if rank != 0:
        return
    prog, seed, groups, bfms, n = make_program(args.config)
    n = args.replicas or n
    times, counted_tot = [], 0
    for i in range(args.warmup + args.steps):
        counted, n_rec, dt, nw, nt = oracle_count_sample(prog)
        if i >= args.warmup:
            times.append(dt)
            counted_tot += counted
    T = sum(times)
    val = counted_tot / T
    line = {"metric": "thread-dyn-instrs profiled/sec and injections/sec at 1/2/4/8 B200 (% HBM roofline)",
            "impl": "reference", "value": val, "unit": "thread-dyn-instrs/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * T / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": workload_name(args.config, n)},
            "cpu_baseline": {"value": val, "unit": "thread-dyn-instrs/s", "cores": nt, "kind": "oracle",
                             "value_per_core": val / nt,
                             "sample": f"each step: oracle golden interpretation + Table II group count of warps "
                                       f"[0,{nw}) of the workload (the cpu_baseline sample of the fi arm)"},
            "e2e": {"value": val, "unit": "thread-dyn-instrs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    # (FI_BENCH_SHARE_GPU=1: ranks share the visible GPUs, e.g. a 2-rank run on a
    # 1-GPU box to exercise the multi-rank path; FI_BENCH_BACKEND=gloo there, since
    # NCCL refuses two ranks on one GPU)
    if os.environ.get("FI_BENCH_SHARE_GPU"):
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        backend = os.environ.get("FI_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    from paper_conf_dsn_0002hsvk21_b200 import fi
    from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign, allreduce_max

    prog, seed, groups, bfms, n = make_program(args.config)
    n = args.replicas or n
    # N > 1: the profile fused with its exchange (fi_profile_peers: chunk rows stored
    # into the peers' memory by the profile kernel itself); FI_BENCH_EXCHANGE=collective
    # for fi_profile + torch.distributed collectives instead
    camp = Campaign(prog, seed, groups, bfms, n, rank, world, dev,
                    exchange=os.environ.get("FI_BENCH_EXCHANGE", "peers"))
    torch.cuda.synchronize()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    clocks = ClockSampler(local)
    clocks.start()                                                # (nvidia-smi needs a moment to start sampling)
    for _ in range(args.warmup):
        camp.step()
    torch.cuda.synchronize()
    camp.check()

    stage_ms = {s: 0.0 for s in STAGES}
    step_ms, prof_ms, inj_ms = [], [], []
    emulated_steps = 0
    if world > 1:
        dist.barrier()
    t_timed0 = time.perf_counter()
    for _ in range(args.steps):
        flush.fill_(1)                                            # L2 flush (256 MiB > 126 MB L2)
        ev = {k: torch.cuda.Event(enable_timing=True) for k in ["start"] + STAGES}
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        camp.step(ev)
        torch.cuda.synchronize()
        prev = "start"
        for s in STAGES:
            stage_ms[s] += ev[prev].elapsed_time(ev[s])
            prev = s
        step_ms.append(ev["start"].elapsed_time(ev["end"]))
        prof_ms.append(ev["start"].elapsed_time(ev["exchange"]))
        inj_ms.append(ev["index"].elapsed_time(ev["classify"]))
        emulated_steps += int(camp.inj_ws[8:16].cpu().view(torch.int64).item())   # K4's own count (fi.h)
    t_timed1 = time.perf_counter()
    time.sleep(0.06)                                              # (the sample in flight at the end)
    clocks.window(t_timed0, t_timed1)
    clk = clocks.stop()
    if world > 1:
        dist.barrier()
    camp.check()

    counts = camp.inst_counts.cpu().numpy().astype(np.uint64)
    counted = int(counts[:, 4].sum() + counts[:, 6].sum())      # NODEST + GPPR = every counted thread-instr
    hist = camp.hist.cpu().numpy()
    assert int(hist.sum()) == n, "histogram does not account for every replica"

    T_total = allreduce_max(sum(step_ms) / 1e3, dev)
    T_prof = allreduce_max((stage_ms["profile"] + stage_ms["exchange"]) / 1e3, dev)
    T_k1 = allreduce_max(stage_ms["profile"] / 1e3, dev)
    T_inj = allreduce_max((stage_ms["select"] + stage_ms["inject"] + stage_ms["classify"]) / 1e3, dev)
    K = args.steps
    # value: the MEDIAN step, each rank's median, max over ranks
    T_prof_med = allreduce_max(statistics.median(prof_ms) / 1e3, dev)
    T_inj_med = allreduce_max(statistics.median(inj_ms) / 1e3, dev)
    value = counted / T_prof_med
    inj_rate = n / T_inj_med

    # K1 roofline: algorithmic bytes per launch = 16 B per record read + 32 B per chunk
    # written + 64 B per instance; duration = CUDA-event profile stage.
    nrec_local = camp.r1 - camp.r0
    nch_local = (camp.r1 - camp.r0 + 1023) // 1024
    algo_bytes = 16 * nrec_local + 32 * nch_local + 64 * camp.dp.n_inst
    k1_ms_local = stage_ms["profile"] / K
    achieved = algo_bytes / (k1_ms_local / 1e3) / 1e9
    peak, peak_src = measured_peaks()
    traffic = None
    tp = os.path.join(ROOT, "profiles", "k1_traffic.json")
    if os.path.exists(tp):
        d = json.load(open(tp))
        if d.get("config") == args.config:
            traffic = d.get("dram_bytes_per_launch")

    # K4 (the dominant kernel of the step) is an emulator: bound by the SM issue rate
    # and memory latency, not HBM bandwidth.  Algorithmic work =
    # the emulated warp-instructions (each needs at least one issue slot natively;
    # K4 counts them itself, fi.h) over its live CUDA-event duration; peak = 148 SMs
    # x 4 schedulers x 1 warp-instruction/clock x the SM clock measured during the
    # run.  sass_* = the SASS warp-instructions K4 actually issues per launch (ncu
    # smsp__inst_executed.sum of the same workload, profiles/k4_counts.json).
    k4_ms_local = stage_ms["inject"] / K
    sm_mhz = clk.get("sm_mhz") or clk.get("sm_max_mhz") or 1965.0
    peak_issue = 148 * 4 * sm_mhz * 1e6
    emu_rate = emulated_steps / K / (k4_ms_local / 1e3)
    k4 = {"bound": "alu", "kernel": "k_inject_jit (K4, JIT-specialised emulator)", "unit": "warp-inst/s",
          "achieved": emu_rate, "peak": peak_issue, "frac": emu_rate / peak_issue, "traffic": None,
          "peak_source": f"148 SMs x 4 SMSPs x 1 issue/clk x {sm_mhz:.0f} MHz (measured SM clock under load)",
          "achieved_is": "emulated warp-instructions per second (K4's own count): one native issue slot each",
          "emulated_warp_steps_per_launch": emulated_steps / K}
    kp = os.path.join(ROOT, "profiles", "k4_counts.json")
    if os.path.exists(kp):
        d = json.load(open(kp))
        if d.get("config") == args.config and d.get("replicas") == n and world == 1 and d.get("kernel") == "k_inject_jit":
            k4["traffic"] = d.get("dram_bytes_per_launch")
            k4["sass_warp_inst_per_s"] = d["sass_warp_inst_per_launch"] / (k4_ms_local / 1e3)
            k4["sass_frac"] = k4["sass_warp_inst_per_s"] / peak_issue
            k4["sass_per_emulated_step"] = d["sass_warp_inst_per_launch"] / max(emulated_steps / K, 1)

    line = {
        "metric": "thread-dyn-instrs profiled/sec and injections/sec at 1/2/4/8 B200 (% HBM roofline)",
        "value": value, "unit": "thread-dyn-instrs/s", "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": 1e3 * T_total / K, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "u32", "data": "synthetic",
        "config": {"workload": workload_name(args.config, n), "records": camp.gt.n_rec, "warps": camp.dp.n_warps,
                   "counted_thread_instrs": counted, "replicas": n, "trace_bytes": 16 * camp.gt.n_rec,
                   "l2": "flushed before every timed step (256 MiB write); trace 39 GB >> 126 MB L2",
                   "parallelism": f"replica+record sharding over {world} GPU(s)"},
        "injections_per_s": inj_rate,
        "value_is": "median over the K timed steps of counted thread-instrs / (profile + count exchange time)",
        "value_mean": counted * K / T_prof, "injections_per_s_mean": n * K / T_inj,
        "stages_ms_per_step": {s: stage_ms[s] / K for s in STAGES},
        "outcomes": {"masked": int(hist[..., 0].sum()), "sdc": int(hist[..., 1].sum()), "due": int(hist[..., 2].sum())},
        "roofline": k4,
        "roofline_profile": {"bound": "hbm", "kernel": "k_profile (K1)", "achieved": achieved, "peak": peak,
                             "unit": "GB/s", "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                             "algorithmic_bytes_per_launch": algo_bytes},
        "clocks": clk,
        # per step: k_profile, 2 x k_scan_rows, k_inst_identities, k_tile_sums, k_select,
        # k_lpt_order, k_inject_jit, k_classify, k_classify_slow
        "gpu_launches": 10 * K,
    }

    if world == 1:
        line["shard_ratio"] = shard_ratio(camp, n)
        line["golden_shards"] = golden_shards(camp.dp)
    if camp.peers is not None:
        camp.peers.close()
    if not args.no_e2e:
        line["e2e"] = e2e(args, prog, seed, groups, bfms, n, rank, world, dev, camp)
    if rank == 0 and world == 1 and not args.no_secondary:
        line["secondary"] = secondary_c4(dev, sm_mhz=clk.get("sm_mhz") or clk.get("sm_max_mhz") or 1965.0)
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(prog, camp.sites_np(), camp)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def shard_ratio(camp, n, G=8, reps=3):
    """North star "near-linear 8-GPU speedup in injections/sec", checked on one GPU:
    the injection stage (select + K4 + K5) of each rank's replica block
    [r*n/G, (r+1)*n/G) timed alone (CUDA events, best of `reps`), against the whole
    set.  The G-GPU stage time is the slowest block; ideal ratio = G."""
    import torch
    from paper_conf_dsn_0002hsvk21_b200 import fi
    from paper_conf_dsn_0002hsvk21_b200.campaign import replica_block
    idx = fi.SiteIndex(camp.gt, camp.inst_counts, camp.chunk_counts, camp.status)

    def stage(j0, m):
        best = None
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fi.select_sites(idx, camp.sched, j0, m, camp.sites, camp.status)
            fi.inject(camp.gt, camp.sites, m, camp.cap, camp.out, camp.log, camp.status, camp.inj_ws, engine="jit")
            h = torch.zeros((8, 4, 3), dtype=torch.int64, device=camp.device)
            fi.classify(camp.gt, camp.sites, m, camp.out, camp.log, camp.cap, h, camp.status)
            b.record()
            torch.cuda.synchronize()
            best = a.elapsed_time(b) if best is None else min(best, a.elapsed_time(b))
        return best
    blocks = [stage(*(lambda j: (j[0], j[1] - j[0]))(replica_block(n, r, G))) for r in range(G)]
    full = stage(0, n)                                # last: camp.sites / out hold the whole set again
    camp.check()
    return {"G": G, "full_ms": full, "block_ms": blocks, "slowest_block_ms": max(blocks),
            "ratio": full / max(blocks), "ideal": G,
            "what": "injection stage (select + K4 + K5) of one rank's replica block [r*n/G,(r+1)*n/G) alone vs all n "
                    "replicas, one GPU, best of 3: the G-GPU injections/s speedup bound"}


def golden_shards(dp, G=8, reps=3):
    """The owner-computes golden run (fi_golden_run_shard) of each rank r of G on
    this GPU, alone: CUDA events around the one C-ABI call (it synchronizes), best
    of `reps` (libfi keeps the device pool's memory mapped between calls).  The G-GPU golden run takes the slowest rank's time."""
    import torch
    from paper_conf_dsn_0002hsvk21_b200 import fi
    if dp.n_inst != 1:
        return None
    def best_of(**kw):
        best = None
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            gt = fi.golden_run(dp, **kw)
            b.record()
            torch.cuda.synchronize()
            best = a.elapsed_time(b) if best is None else min(best, a.elapsed_time(b))
            del gt
        return best
    full = best_of()                      # (the first call also maps the pool the later calls reuse)
    out = [best_of(rank=r, world=G) for r in range(G)]
    return {"G": G, "full_ms": full, "rank_ms": out, "slowest_rank_ms": max(out), "ratio": full / max(out),
            "what": "owner-computes golden run (fi_golden_run_shard: sliced pass 1 of all warps, pass 2 of the rank's "
                    "record shard) of each rank alone on one GPU vs the whole golden run (fi_golden_run)"}


def secondary_c4(dev, n=256, sm_mhz=1965.0):
    """BASELINE configs[3]'s program (ResNet-50 v1.5 inference shape, 72 launches)
    on one GPU: golden run, exact profile, select, K4, K8 whole-program outcomes
    for a bounded replica sample (the 100 k campaign shards these over ranks).
    CUDA events on the launching stream; not part of `value`."""
    import torch
    from fi_inputs import resnet as R
    from paper_conf_dsn_0002hsvk21_b200 import fi
    import time as _t
    prog = R.c4(full=True)
    dp = fi.DeviceProgram(prog, dev)
    t0 = _t.perf_counter()
    dp.jit(fi.FI_JIT_INJECT | fi.FI_JIT_GOLDEN | fi.FI_JIT_PAGE)     # one module per static kernel, compiled in parallel
    jit_s = _t.perf_counter() - t0
    torch.cuda.synchronize()
    t0 = _t.perf_counter()
    gt = fi.golden_run(dp, engine="jit")
    torch.cuda.synchronize()
    golden_s = _t.perf_counter() - t0
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(5)]
    cap = fi.log_capacity(gt)
    idx = sites = out = log = hist = None
    k8_steps = []
    for rep in range(2):                                            # the first pass warms allocations
        idx = sites = out = log = hist = None                      # (freed, so the second pass reuses them)
        torch.cuda.synchronize()
        ev[0].record()
        ic, cc = fi.profile(gt)
        ev[1].record()
        idx = fi.SiteIndex(gt, ic, cc)
        sites = fi.select_sites(idx, fi.schedule(R.C4_CAMPAIGN_SEED, [fi.G_GP], [0]), 0, n)
        ev[2].record()
        out, log = fi.inject(gt, sites, n, cap, engine="jit")
        ev[3].record()
        # (the warm-up pass also reads back K8's emulated-step count: the same work both passes)
        hist = fi.classify_batched(gt, sites, n, out, log, cap, engine="jit", steps_out=k8_steps if rep == 0 else None)
        ev[4].record()
        torch.cuda.synchronize()
    ms = [ev[i].elapsed_time(ev[i + 1]) for i in range(4)]
    counts = ic.cpu().numpy()
    counted = int(counts[:, 4].sum() + counts[:, 6].sum())
    h = hist.cpu().numpy()
    return {"workload": "C4 ResNet-50 v1.5 inference, 224x224, batch 1: 72 launches, 265,696 warps; "
                        f"{n} replicas G_GP FLIP_SINGLE_BIT, whole-program outcomes (K8)",
            "records": gt.n_rec, "profile_thread_instrs_per_s": counted / (ms[0] / 1e3),
            "injections_per_s": n / ((ms[1] + ms[2] + ms[3]) / 1e3),
            "ms": {"profile": ms[0], "index_select": ms[1], "inject_k4": ms[2], "propagate_classify_k8": ms[3]},
            "outcomes": {"masked": int(h[..., 0].sum()), "sdc": int(h[..., 1].sum()), "due": int(h[..., 2].sum())},
            "engine": "jit", "jit_compile_s": jit_s, "golden_run_s": golden_s,
            "roofline_k8": k8_roofline(k8_steps[0] if k8_steps else 0, ms[3], sm_mhz)}


def k8_roofline(steps, k8_ms, sm_mhz=1965.0):
    """K8 (fi_classify_batched_jit) against the SM issue-slot roofline of §7.2: the
    emulated warp-instructions of every re-executed warp (K8 counts them, fi.h)
    per second of the WHOLE call — exec plus the end-of-launch fix-ups, so a
    conservative figure for k8_exec_jit alone."""
    peak = 148 * 4 * sm_mhz * 1e6
    ach = steps / (k8_ms / 1e3) if k8_ms > 0 else 0.0
    return {"bound": "alu", "kernel": "k8_exec_jit + end-of-launch fix-ups (the whole K8 call)", "unit": "warp-inst/s",
            "achieved": ach, "peak": peak, "frac": ach / peak, "emulated_warp_steps": steps,
            "peak_source": f"148 SMs x 4 SMSPs x 1 issue/clk x {sm_mhz:.0f} MHz (the SM clock sampled in the timed region)"}


def e2e(args, prog, seed, groups, bfms, n, rank, world, dev, camp):
    """End to end through the public API — ONE fi_campaign call (C ABI) from HOST
    buffers: H2D of the program (pinned), golden run (both passes), profile,
    count exchange, index, select, inject, classify, histogram exchange, D2H of
    histogram + per-replica sites and results; CUDA events inside fi_campaign,
    wall clock around the call (synchronous), max over ranks."""
    import torch
    from paper_conf_dsn_0002hsvk21_b200 import fi
    from paper_conf_dsn_0002hsvk21_b200.campaign import allreduce_max
    host = {k: torch.from_numpy(np.ascontiguousarray(getattr(prog, k)).view(np.uint8).reshape(-1).copy()).pin_memory()
            for k in ("code", "kernels", "instances", "cbank", "buffers", "init_image")}
    # bytes fi_campaign moves host -> device: the tables, and the image minus the
    # buffers with a writer (zeroed on the device), gaps < 1 MiB merged
    h2d = sum(host[k].numel() for k in ("code", "kernels", "instances", "cbank", "buffers"))
    rng = []
    for b in prog.buffers:
        if int(b["writer"]) >= 0 or not int(b["size"]):
            continue
        o, e = int(b["off"]), int(b["off"]) + int(b["size"])
        if rng and o >= rng[-1][1] and o - rng[-1][1] < (1 << 20):
            rng[-1][1] = max(rng[-1][1], e)
        else:
            rng.append([o, e])
    h2d += sum(e - o for o, e in rng)
    del camp
    torch.cuda.empty_cache()
    # start from an empty device pool (golden_shards' runs left theirs mapped): the
    # first call maps what the campaign needs, the timed calls reuse it
    fi.campaign_release_memory(dev.index if dev.index is not None else -1)
    times, r, jit_ms = [], None, []
    for it in range(4):
        if world > 1:
            import torch.distributed as dist
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = fi.campaign(prog, seed, groups, bfms, n, rank, world, host=host, engine="jit",
                        owner_computes=(world > 1 and len(prog.instances) == 1))
        times.append(time.perf_counter() - t0)
        jit_ms.append(r.ms["jit"])
    fi.campaign_release_memory(dev.index if dev.index is not None else -1)
    assert int(r.hist.sum()) == n
    n_loc = r.n_local
    d2h = r.hist.nbytes + n_loc * (fi.SITE_DTYPE.itemsize + fi.INJ_DTYPE.itemsize) + r.inst_counts.nbytes
    T = allreduce_max(min(times[1:]), dev)
    return {"value": r.counted / T, "unit": "thread-dyn-instrs/s", "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": d2h, "injections_per_s": n / T, "seconds": T,
            "api": "fi_campaign (C ABI) via paper_conf_dsn_0002hsvk21_b200.fi.campaign, K4 engine JIT",
            "cold_seconds": times[0], "jit_compile_s": jit_ms[0] / 1e3,
            "timing": "value/seconds: the fastest of calls 2-4 (JIT module cached in-process and device memory "
                      "kept in the pool by the first call, which reports cold_seconds including the one-time NVRTC "
                      "compile and the first allocations)", "warm_seconds": times[1:],
            "stages_ms": r.ms,
            "includes": "H2D program+image (pinned), golden run passes 1+2 (trace generation + checkpoints), "
                        "profile, count exchange, index, select, inject, classify, histogram exchange, "
                        "D2H histogram+sites+results+counts"}


if __name__ == "__main__":
    main()
