"""GPU parity of fi_campaign — the whole campaign of one rank through ONE C-ABI
call from host arrays (golden run, sharded profile, count exchange, index,
select, inject, classify, histogram exchange) — against the CPU oracle, and its
sharded path (world = 2 and 3 on one GPU, ranks as threads, the all-reduce
callback summing on the host) against world = 1: bit-identical sites, injected
values and outcomes, identical histograms."""
import threading

import numpy as np
import pytest
import torch

import oracle as O
from fi_inputs import programs as P

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    from paper_conf_dsn_0002hsvk21_b200 import fi
    return fi


def _site_rows(a):
    return np.stack([a[n].astype(np.uint64) for n in a.dtype.names], axis=1)


def _check_vs_oracle(F, prog, r, seed, groups, bfms, n, approximate=False):
    g = O.Golden(prog)
    if approximate:
        os_ = g.select_approx(seed, groups, bfms, 0, n)
    else:
        os_ = g.select(seed, groups, bfms, 0, n)
        assert np.array_equal(r.inst_counts[: len(prog.instances)], g.counts())
        c = g.counts()
        assert r.counted == int(c[:, 4].sum() + c[:, 6].sum())
    assert r.n_rec == g.n_records
    assert np.array_equal(_site_rows(r.sites), _site_rows(os_))
    oi = g.inject(os_, O.MODE_FULL)
    for f in ("outcome", "flags"):
        assert np.array_equal(r.inj[f], oi[f]), f
    ok = os_["flags"] == 0
    for f in ("before", "after", "mask", "fault_kind"):
        assert np.array_equal(r.inj[f][ok], oi[f][ok]), f
    assert np.array_equal(r.hist, O.histogram(os_, oi))
    return oi


def test_campaign_c1(F):
    prog = P.c1()
    r = F.campaign(prog, P.CAMPAIGN_SEED[1], [F.G_GP], [0], 100)
    _check_vs_oracle(F, prog, r, P.CAMPAIGN_SEED[1], [F.G_GP], [0], 100)
    assert r.totals[F.G_GP] == 14336 and r.n_local == 100 and r.j0 == 0
    assert r.ms["golden"] > 0 and r.ms["inject"] > 0


@pytest.mark.parametrize("prop", ["k7", "k8", "auto"])
def test_campaign_chain_propagation(F, prop):
    prog = P.multi_instance_chain(6, shrink=29)
    seed, groups, bfms = 0x7A7, [F.G_GP, F.G_LD, F.G_FP32], [0, 1, 2, 3]
    r = F.campaign(prog, seed, groups, bfms, 300, propagation=prop, ckpt=0)
    oi = _check_vs_oracle(F, prog, r, seed, groups, bfms, 300)
    assert (oi["outcome"] == O.SDC).sum() > 0


def test_campaign_unchecked_approximate(F):
    prog = P.multi_instance_chain(n_inst=6, n=256, shrink=33)
    seed, groups, bfms = 0xA11, [F.G_GP, F.G_FP32, F.G_LD], [0, 1, 2, 3]
    r = F.campaign(prog, seed, groups, bfms, 400, approximate=True)
    _check_vs_oracle(F, prog, r, seed, groups, bfms, 400, approximate=True)
    assert r.n_not_injected == int((r.sites["flags"] == 1).sum()) > 0


class _HostAllReduce:
    """World-size-w all-reduce for ranks running as threads on one GPU: each rank
    copies its device integers to the host, the last one in sums, all copy back."""

    def __init__(self, world, F):
        self.world, self.F = world, F
        self.bar = threading.Barrier(world)
        self.parts = {}
        self.calls = 0

    def fn(self, rank):
        F = self.F

        def cb(dev, count, elem_bytes, ctx, stream):
            try:
                d = torch.device("cuda", torch.cuda.current_device())
                s = torch.cuda.ExternalStream(stream, device=d)
                t = F.device_view(dev, count, elem_bytes, d)
                with torch.cuda.stream(s):
                    self.parts[rank] = t.cpu()
                self.bar.wait()
                tot = sum(self.parts[r] for r in range(self.world))
                self.bar.wait()
                with torch.cuda.stream(s):
                    t.copy_(tot.to(d))
                s.synchronize()
                if rank == 0:
                    self.calls += 1
                return 0
            except Exception as e:                       # pragma: no cover
                print("allreduce failed", e)
                self.bar.abort()
                return 1
        return F.ALLREDUCE_FN(cb)


def _run_world(F, prog, seed, groups, bfms, n, world, **kw):
    ar = _HostAllReduce(world, F)
    cbs = [ar.fn(r) for r in range(world)]
    out = [None] * world
    err = []

    def body(r):
        try:
            torch.cuda.set_device(0)
            out[r] = F.campaign(prog, seed, groups, bfms, n, rank=r, world=world, allreduce=cbs[r], **kw)
        except Exception as e:
            err.append(e)
            ar.bar.abort()
    ths = [threading.Thread(target=body, args=(r,)) for r in range(world)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    assert not err, err
    return out, ar.calls


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("maker,prop", [(P.c1, "auto"), (lambda: P.c2(full=False), "auto"),
                                        (lambda: P.multi_instance_chain(6, shrink=29), "k8")])
def test_campaign_sharded_equals_single(F, world, maker, prop):
    prog = maker()
    seed, groups, bfms, n = 0x5EED, [F.G_GP, F.G_LD], [0, 1, 2, 3], 240
    one = F.campaign(prog, seed, groups, bfms, n, propagation=prop)
    parts, calls = _run_world(F, prog, seed, groups, bfms, n, world, propagation=prop)
    assert calls == 1                                      # the histogram (the profile is the golden run's own)
    assert [p.j0 for p in parts] == [n * r // world for r in range(world)]
    assert sum(p.n_local for p in parts) == n
    assert parts[0].rec_range[0] == 0 and parts[-1].rec_range[1] == one.n_rec
    for a, b in zip(parts, parts[1:]):
        assert a.rec_range[1] == b.rec_range[0] and a.rec_range[1] % 1024 == 0
    for p in parts:
        assert np.array_equal(p.hist, one.hist)
        assert np.array_equal(p.inst_counts, one.inst_counts)
        assert p.totals == one.totals
    sites = np.concatenate([p.sites for p in parts])
    inj = np.concatenate([p.inj for p in parts])
    assert np.array_equal(_site_rows(sites), _site_rows(one.sites))
    assert np.array_equal(inj.view(np.uint8), one.inj.view(np.uint8))


def test_campaign_errors(F):
    prog = P.c1()
    with pytest.raises(F.FIError) as e:
        F.campaign(prog, 1, [F.G_NODEST], [0], 10)
    assert e.value.code == F.FI_E_NOT_INJECTABLE
    prog0 = P.vector_add(n=64)
    with pytest.raises(F.FIError) as e:
        F.campaign(prog0, 1, [F.G_FP64], [0], 10)
    assert e.value.code == F.FI_E_EMPTY_GROUP


def test_campaign_repeat_reuses_pool_then_release(F):
    """fi_campaign's device memory comes from the device's default pool and stays
    reserved between calls: a repeated campaign gives identical results, and
    fi_campaign_release_memory hands the memory back."""
    prog = P.c2(full=False)
    r1 = F.campaign(prog, 11, [F.G_GP], [0, 1, 2, 3], 64)
    r2 = F.campaign(prog, 11, [F.G_GP], [0, 1, 2, 3], 64)
    assert np.array_equal(r1.hist, r2.hist)
    assert np.array_equal(_site_rows(r1.sites), _site_rows(r2.sites))
    assert np.array_equal(r1.inj["outcome"], r2.inj["outcome"])
    F.campaign_release_memory()
    r3 = F.campaign(prog, 11, [F.G_GP], [0, 1, 2, 3], 64)
    assert np.array_equal(r1.hist, r3.hist)


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("maker", [P.c1, lambda: P.c2(full=False), lambda: P.fuzz_program(4),
                                   lambda: P.vector_add(n=1000)])
def test_campaign_owner_computes_equals_single(F, world, maker):
    """Owner-computes: each rank runs the golden pass 2 of its own
    record shard's warps only, the golden image is completed by one SUM over the
    writer buffers, and a rank injects exactly the replicas whose site lies in
    its shard.  Every replica appears on exactly one rank, bit-identical to the
    world-1 campaign; histograms and counts identical."""
    prog = maker()
    seed, groups, bfms, n = 0x0C0C, [F.G_GP, F.G_LD], [0, 1, 2, 3], 300
    one = F.campaign(prog, seed, groups, bfms, n)
    parts, calls = _run_world(F, prog, seed, groups, bfms, n, world, owner_computes=True)
    assert calls == 4                                      # golden image, inst_counts, chunk_counts, histogram
    j = np.concatenate([p.j for p in parts])
    assert np.array_equal(np.sort(j), np.arange(n))       # each replica on exactly one rank
    order = np.argsort(j)
    sites = np.concatenate([p.sites for p in parts])[order]
    inj = np.concatenate([p.inj for p in parts])[order]
    assert np.array_equal(_site_rows(sites), _site_rows(one.sites))
    assert np.array_equal(inj.view(np.uint8), one.inj.view(np.uint8))
    for p in parts:
        assert np.array_equal(p.hist, one.hist)
        assert np.array_equal(p.inst_counts, one.inst_counts)
        assert p.totals == one.totals
        lo, hi = p.rec_range                               # its sites lie in its record shard
        w0 = np.asarray(p.sites["warp"])
        assert len(w0) == 0 or (p.n_local == len(p.j))
