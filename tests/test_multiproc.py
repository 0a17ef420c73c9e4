"""The N>1 path on CPU: world-size-2 gloo process groups running the campaign's
host-side sharding and its collectives (campaign.record_shard, replica_block,
allreduce_sum_, allreduce_max).  Per-rank partial results come from the oracle's
trace (brute-force per-record sums), so the check is that sharded + reduced
equals unsharded, bit for bit, for any world size."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from fi_inputs import programs as P
from paper_conf_dsn_0002hsvk21_b200.campaign import (allgather_chunks_, allreduce_max, allreduce_sum_, record_shard,
                                                     replica_block)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _partial_counts(trace, r0, r1, n_inst):
    c = np.zeros((n_inst, 8), dtype=np.int64)
    chunks = np.zeros(((len(trace) + 1023) // 1024, 8), dtype=np.int32)
    for r in range(r0, r1):
        rec = trace[r]
        n = bin(int(rec["active"]) & int(rec["pred"])).count("1")
        gm = int(rec["insn"]) >> 24
        for g in range(8):
            if (gm >> g) & 1:
                c[int(rec["instance"]), g] += n
                chunks[r // 1024, g] += n
    return c, chunks


def _worker(rank, world, port, prog_name, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    prog = {"mini": lambda: P.sgemm(128, 256, 16), "chain": lambda: P.multi_instance_chain(5)}[prog_name]()
    g = O.Golden(prog, n_threads=1)
    t = g.trace()
    r0, r1 = record_shard(len(t), rank, world)
    c, ch = _partial_counts(t, r0, r1, len(prog.instances))
    ct, cht = torch.from_numpy(c), torch.from_numpy(ch)
    chg = cht.clone()
    allreduce_sum_(ct)
    allreduce_sum_(cht)
    allgather_chunks_(chg, len(t))                   # the bench's exchange: all-gather of the owned rows
    # replica block of a small campaign, oracle outcomes, histogram all-reduce
    n = 37
    j0, j1 = replica_block(n, rank, world)
    sites = g.select(0xC0000002, [7, 3], [0, 1, 2, 3], j0, j1 - j0)
    inj = g.inject(sites, O.MODE_FULL, n_threads=1)
    h = torch.from_numpy(O.histogram(sites, inj).astype(np.int64))
    allreduce_sum_(h)
    mx = allreduce_max(float(rank + 1), "cpu")
    if rank == 0:
        full_sites = g.select(0xC0000002, [7, 3], [0, 1, 2, 3], 0, n)
        full_hist = O.histogram(full_sites, g.inject(full_sites, O.MODE_FULL, n_threads=1))
        fc, fch = _partial_counts(t, 0, len(t), len(prog.instances))
        q.put(dict(counts_ok=bool((ct.numpy() == fc).all() and (ct.numpy().astype(np.uint64) == g.counts()).all()),
                   chunks_ok=bool((cht.numpy() == fch).all() and (chg.numpy() == fch).all()),
                   hist_ok=bool((h.numpy() == full_hist.astype(np.int64)).all()),
                   max_ok=(mx == float(world))))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,prog_name", [(2, "mini"), (2, "chain"), (3, "mini")])
def test_sharded_equals_unsharded(world, prog_name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, prog_name, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert res == dict(counts_ok=True, chunks_ok=True, hist_ok=True, max_ok=True)


def test_partitions_cover_exactly():
    for n in (0, 1, 7, 10000, 10001):
        for w in (1, 2, 3, 4, 8):
            blocks = [replica_block(n, r, w) for r in range(w)]
            assert blocks[0][0] == 0 and blocks[-1][1] == n
            assert all(blocks[i][1] == blocks[i + 1][0] for i in range(w - 1))
            assert max(b - a for a, b in blocks) - min(b - a for a, b in blocks) <= 1
    for n_rec in (0, 1, 1023, 1024, 1025, 2449850368):
        for w in (1, 2, 4, 8):
            sh = [record_shard(n_rec, r, w) for r in range(w)]
            assert sh[0][0] == 0 and sh[-1][1] == n_rec
            assert all(sh[i][1] == sh[i + 1][0] for i in range(w - 1))
            assert all(a % 1024 == 0 for a, _ in sh)
