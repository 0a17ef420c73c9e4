"""Owner-computes multi-GPU campaigns on CPU: the host-side
partition libfi computes (fi_shard_warps) and, at world size 2 and 3 over gloo,
the campaign split it implies — every rank draws all replicas and keeps those
whose site lies in its record shard — against the unsharded campaign, with the
oracle standing in for the GPU stages.  The GPU path of the same split is
tests/test_gpu_campaign.py::test_campaign_owner_computes_equals_single."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from fi_inputs import programs as P
from paper_conf_dsn_0002hsvk21_b200 import fi
from paper_conf_dsn_0002hsvk21_b200.campaign import allreduce_sum_, record_shard


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_shard_warps_partition(seed, world):
    rng = np.random.Generator(np.random.PCG64(seed))
    W = int(rng.integers(1, 300))
    lens = rng.integers(0, 5000, W).astype(np.uint64)
    lens[rng.random(W) < 0.2] = 0                         # empty warps (a whole CTA past n, say)
    woff = np.concatenate([[0], np.cumsum(lens)]).astype(np.uint64)
    n_rec = int(woff[-1])
    owned = np.zeros(W, dtype=int)
    prev_end = 0
    for r in range(world):
        sh = fi.shard_warps(woff, r, world)
        r0, r1 = sh["rec"]
        assert (r0, r1) == record_shard(n_rec, r, world)              # = fi_campaign's profile shard
        assert r0 == prev_end
        prev_end = r1
        wa, wb = sh["run"]
        oa, ob = sh["own"]
        for w in range(W):
            a, b = int(woff[w]), int(woff[w + 1])
            overlaps = a < b and a < r1 and b > r0
            if overlaps:
                assert wa <= w < wb, (w, sh)                 # pass 2 runs every warp holding shard records
            elif wa <= w < wb:
                assert a == b                                # ... and no other warp with records
            if oa <= w < ob and a < b:
                owned[w] += 1
                assert r0 <= a < r1 and wa <= w < wb         # an owner runs its warp
    assert prev_end == n_rec
    assert (owned[lens > 0] == 1).all()                      # every warp with records has exactly one owner


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    prog = P.sgemm(128, 256, 16)
    g = O.Golden(prog, n_threads=1)
    woff = np.concatenate([[0], np.cumsum(g.warp_len())]).astype(np.uint64)
    sh = fi.shard_warps(woff, rank, world)
    r0, r1 = sh["rec"]
    n, seed, groups, bfms = 53, 0xC0000002, [O.G_GP, O.G_LD], [0, 1, 2, 3]
    drawn = g.select(seed, groups, bfms, 0, n)                # every rank draws every replica
    rec = woff[drawn["warp"]] + drawn["step"]
    mine = (rec >= r0) & (rec < r1)
    w = drawn["warp"][mine]
    assert ((w >= sh["run"][0]) & (w < sh["run"][1])).all()  # its sites' warps are the ones it emulated
    inj = g.inject(drawn[mine], O.MODE_FULL, n_threads=1)
    h = torch.from_numpy(O.histogram(drawn[mine], inj).astype(np.int64))
    allreduce_sum_(h)
    cnt = torch.zeros(n, dtype=torch.int64)
    cnt[torch.from_numpy(np.flatnonzero(mine))] = 1
    allreduce_sum_(cnt)
    if rank == 0:
        full = g.inject(drawn, O.MODE_FULL, n_threads=1)
        q.put(dict(hist_ok=bool((h.numpy() == O.histogram(drawn, full).astype(np.int64)).all()),
                   each_once=bool((cnt.numpy() == 1).all())))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_owner_split_equals_unsharded(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert res == dict(hist_ok=True, each_once=True)
