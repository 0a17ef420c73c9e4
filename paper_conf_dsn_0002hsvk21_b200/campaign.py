"""Campaign driver: one process per GPU, torch.distributed (NCCL) for the two
exchanges the path has:

  1. after the sharded profile: all_reduce(SUM) of inst_counts [K][8] (u64 as
     int64) and an all-gather of chunk_counts [C][8] (each rank filled only its own chunks,
     so the sum is an all-gather);
  2. at the end: all_reduce(SUM) of the outcome histogram [8][4][3].

Both are integer sums, so results are bit-identical for any world size; the
replica RNG is keyed by the GLOBAL replica index j, so every
replica's site, injection and outcome are independent of the GPU count.
The paper runs one injection per OS process [PAPER.md:244]; here a rank runs a
contiguous block of replicas [r*n/G, (r+1)*n/G) as independent warps.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

FI_CHUNK = 1024


# ---- host-side partitioning (pure, tested on CPU) ---------------------------
def record_shard(n_rec: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous record range of rank r, aligned to 1,024-record chunks."""
    n_chunks = (n_rec + FI_CHUNK - 1) // FI_CHUNK
    c0 = n_chunks * rank // world
    c1 = n_chunks * (rank + 1) // world
    return min(c0 * FI_CHUNK, n_rec), min(c1 * FI_CHUNK, n_rec)


def replica_block(n: int, rank: int, world: int) -> tuple[int, int]:
    return n * rank // world, n * (rank + 1) // world


def allreduce_sum_(t: torch.Tensor, group=None) -> torch.Tensor:
    """In-place integer SUM across ranks (no-op when not distributed)."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t


def allgather_chunks_(cc: torch.Tensor, n_rec: int, group=None) -> torch.Tensor:
    """In place: every rank's chunk_counts rows [c0_r, c1_r) (its record shard,
    record_shard) gathered into every rank's [C][8] array — the same result as the
    SUM all-reduce (each rank wrote only its own chunks, the rest are zero) with
    half the bytes of a ring all-reduce: rank slices padded to ceil(C/G) rows,
    one all_gather_into_tensor, then the slices copied into place."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return cc
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    if world == 1:
        return cc
    C = cc.shape[0]
    per = (C + world - 1) // world
    bounds = [(C * r // world, C * (r + 1) // world) for r in range(world)]
    c0, c1 = bounds[rank]
    send = torch.zeros((per,) + tuple(cc.shape[1:]), dtype=cc.dtype, device=cc.device)
    send[: c1 - c0] = cc[c0:c1]
    recv = torch.empty((world * per,) + tuple(cc.shape[1:]), dtype=cc.dtype, device=cc.device)
    dist.all_gather_into_tensor(recv, send, group=group)
    for r, (a, b) in enumerate(bounds):
        if r != rank and b > a:
            cc[a:b] = recv[r * per: r * per + (b - a)]
    assert (n_rec + FI_CHUNK - 1) // FI_CHUNK == C
    return cc


def allreduce_max(x: float, device, group=None) -> float:
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        t = torch.tensor([x], dtype=torch.float64, device=device)
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        return float(t.item())
    return x


@dataclass
class StepResult:
    hist: torch.Tensor
    inst_counts: torch.Tensor
    n_replicas: int
    stage_ms: dict = field(default_factory=dict)


class Campaign:
    """Golden run + per-step profile / index / select / inject / classify for one
    program on this rank's GPU (all work in libfi kernels)."""

    def __init__(self, prog, seed: int, groups, bfms, n_replicas: int, rank: int = 0, world: int = 1,
                 device="cuda", group=None, host_tensors: dict | None = None, propagation: str = "auto",
                 engine: str = "jit", exchange: str = "collective"):
        """propagation: how a multi-launch program's outcome is computed — "k7"
        (fi_classify: one CUDA warp walks a replica's later launches), "k8"
        (fi_classify_batched: replica batches in lockstep over the launches), or
        "auto" (K8 from 64 launches on).  Both give identical results.
        engine: "jit" (golden passes, K4 and K8 on the program's JIT module, built
        once here) or "interp" (the shared-memory interpreter); identical results.
        exchange (world > 1): "collective" (fi_profile, then torch.distributed
        all-reduce / all-gather) or "peers" (fi_profile_peers: the profile kernel
        stores its chunk rows straight into the peers' memory over NVLink and the
        ranks synchronise on device flags — no separate collective); identical results."""
        from . import fi
        self.fi = fi
        self.prog = prog
        self.rank, self.world, self.group = rank, world, group
        self.device = torch.device(device)
        self.sched = fi.schedule(seed, groups, bfms)
        self.n = n_replicas
        self.j0, self.j1 = replica_block(n_replicas, rank, world)
        self.dp = fi.DeviceProgram(prog, self.device, host_tensors)
        self.engine = engine
        self.batched = propagation == "k8" or (propagation == "auto" and self.dp.n_inst >= 64)
        if engine == "jit":
            self.dp.jit(fi.FI_JIT_INJECT | fi.FI_JIT_GOLDEN | (fi.FI_JIT_PAGE if self.batched else 0))
        self.gt = fi.golden_run(self.dp, engine=engine)
        self.r0, self.r1 = record_shard(self.gt.n_rec, rank, world)
        self.cap = fi.log_capacity(self.gt)
        nloc = max(self.j1 - self.j0, 1)
        K, C = self.dp.n_inst, max(self.gt.n_chunks, 1)
        self.inst_counts = torch.zeros((K, 8), dtype=torch.int64, device=self.device)
        self.chunk_counts = torch.zeros((C, 8), dtype=torch.int32, device=self.device)
        self.peers = None
        if exchange == "peers" and world > 1:
            self.peers = fi.PeerExchange(C, K, rank, world, self.device, group)
            self.chunk_counts = self.peers.chunk_counts   # (its rows arrive from the peers' profile kernels)
        elif exchange not in ("collective", "peers"):
            raise ValueError(exchange)
        self.sites = torch.empty(nloc * 64, dtype=torch.uint8, device=self.device)
        self.out = torch.empty(nloc * 24, dtype=torch.uint8, device=self.device)
        self.log = torch.empty(nloc * self.cap * 16, dtype=torch.uint8, device=self.device)
        self.hist = torch.zeros((8, 4, 3), dtype=torch.int64, device=self.device)
        self.status = fi.DeviceStatus(self.device)
        self.inj_ws = torch.empty(fi.lib().fi_inject_workspace(nloc), dtype=torch.uint8, device=self.device)

    @property
    def n_local(self):
        return self.j1 - self.j0

    def step(self, events: dict | None = None) -> StepResult:
        fi = self.fi
        ev = events if events is not None else {}

        def mark(name):
            if name in ev:
                ev[name].record()

        mark("start")
        if self.peers is not None:
            # K1 with its rows stored into every peer, partial counts pushed, device-side
            # flag wait, partial sum: one stream-ordered call, the exchange inside it
            self.peers.profile(self.gt, self.r0, self.r1, self.inst_counts, self.status)
            mark("profile")
        else:
            if self.world > 1:
                self.chunk_counts.zero_()
            fi.profile(self.gt, self.r0, self.r1, self.inst_counts, self.chunk_counts)
            mark("profile")
            if self.world > 1:
                allreduce_sum_(self.inst_counts, self.group)
                allgather_chunks_(self.chunk_counts, self.gt.n_rec, self.group)
        mark("exchange")
        idx = fi.SiteIndex(self.gt, self.inst_counts, self.chunk_counts, self.status)
        mark("index")
        n = self.n_local
        fi.select_sites(idx, self.sched, self.j0, n, self.sites, self.status)
        mark("select")
        fi.inject(self.gt, self.sites, n, self.cap, self.out, self.log, self.status, self.inj_ws, engine=self.engine)
        mark("inject")
        self.hist.zero_()
        if self.batched:
            fi.classify_batched(self.gt, self.sites, n, self.out, self.log, self.cap, self.hist, status=self.status,
                                engine=self.engine)
        else:
            fi.classify(self.gt, self.sites, n, self.out, self.log, self.cap, self.hist, self.status)
        mark("classify")
        allreduce_sum_(self.hist, self.group)
        mark("end")
        return StepResult(self.hist, self.inst_counts, self.n)

    def check(self):
        self.status.check("campaign step")

    def sites_np(self):
        return self.fi.as_numpy(self.sites, self.fi.SITE_DTYPE, self.n_local)

    def inj_np(self):
        return self.fi.as_numpy(self.out, self.fi.INJ_DTYPE, self.n_local)


def summarize(hist: np.ndarray) -> dict:
    """Outcome shares with the PAPER.md:214 worst-case margins."""
    import math
    tot = hist.sum()
    res = {}
    for i, name in enumerate(("masked", "sdc", "due")):
        c = int(hist[..., i].sum())
        p = c / tot if tot else 0.0
        res[name] = {"count": c, "share": p, "ci95": 1.959963984540054 * math.sqrt(p * (1 - p) / max(tot, 1))}
    return res
