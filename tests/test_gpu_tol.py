"""C-12 secondary numeric classification on the GPU (rtol = 1e-6, atol = 0,
NaN != number) against the oracle, whose
tolerance mode is pinned to numpy in tests/test_oracle_tol.py.  Every
classifier: K5 (single launch: fast path, slow path, f64 element partner
lookups), K7 (overlay), K8 (dense compare of the remaining output pages;
interpreter and JIT re-execution), and fi_campaign's hist_tol.  The graded
bitwise outcome must not change with rtol."""
import numpy as np
import pytest

import oracle as O
from fi_inputs import programs as P

pytestmark = pytest.mark.gpu
RTOL = 1e-6


@pytest.fixture(scope="module")
def F():
    from paper_conf_dsn_0002hsvk21_b200 import fi
    return fi


def _campaign(F, prog, seed, groups, bfms, n, how):
    g = O.Golden(prog)
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    ic, cc = F.profile(gt)
    sites = F.select_sites(F.SiteIndex(gt, ic, cc), F.schedule(seed, groups, bfms), 0, n)
    os_ = g.select(seed, groups, bfms, 0, n)
    cap = F.log_capacity(gt)
    out, log = F.inject(gt, sites, n, cap)
    out0, log0 = out.clone(), log.clone()          # (K7 reuses a replica's K4 log as scratch)
    import torch
    hist_tol = torch.zeros((8, 4, 3), dtype=torch.int64, device=dp.device)
    if how == "k5k7":
        hist = F.classify(gt, sites, n, out, log, cap, rtol=RTOL, hist_tol=hist_tol)
        hist0 = F.classify(gt, sites, n, out0, log0, cap)
    else:
        engine = "jit" if how == "k8jit" else "interp"
        hist = F.classify_batched(gt, sites, n, out, log, cap, rtol=RTOL, hist_tol=hist_tol, engine=engine)
        hist0 = F.classify_batched(gt, sites, n, out0, log0, cap, engine=engine)
    gi = F.as_numpy(out, F.INJ_DTYPE, n)
    g0 = F.as_numpy(out0, F.INJ_DTYPE, n)
    oi = g.inject(os_, O.MODE_FULL, rtol=RTOL)
    for f in ("outcome", "flags", "fault_kind"):
        bad = np.flatnonzero(gi[f] != oi[f])
        assert bad.size == 0, f"{f}: replica {bad[0]} gpu {gi[bad[0]]} oracle {oi[bad[0]]}"
    assert (g0["outcome"] == gi["outcome"]).all()                         # graded class unchanged
    assert ((g0["flags"] & F.FI_SDC_WITHIN_TOL) == 0).all()
    assert np.array_equal(hist.cpu().numpy(), hist0.cpu().numpy())
    assert np.array_equal(hist.cpu().numpy().astype(np.uint64), O.histogram(os_, oi))
    assert np.array_equal(hist_tol.cpu().numpy().astype(np.uint64), O.histogram(os_, oi, tol=True))
    return oi


@pytest.mark.parametrize("maker,groups", [
    (P.c1, [O.G_GP, O.G_FP32, O.G_LD]),
    (P.vector_add_f64, [O.G_GP, O.G_FP64, O.G_LD]),
    (lambda: P.c2(full=False), [O.G_GP]),
    (lambda: P.fuzz_program(3), [O.G_GP, O.G_GPPR]),
])
def test_k5_single_launch(F, maker, groups):
    oi = _campaign(F, maker(), 0x70150, groups, [0, 1, 2, 3], 600, "k5k7")
    within = (oi["outcome"] == O.SDC) & ((oi["flags"] & O.SDC_WITHIN_TOL) != 0)
    if maker in (P.c1, P.vector_add_f64):
        assert within.any() and ((oi["outcome"] == O.SDC) & ~within).any()


@pytest.mark.parametrize("how", ["k5k7", "k8", "k8jit"])
@pytest.mark.parametrize("maker,groups", [(lambda: P.multi_instance_chain(5), [O.G_GP, O.G_FP32, O.G_LD]),
                                          (P.scatter_chain, [O.G_GP, O.G_LD]),
                                          (lambda: P.c3(full=False), [O.G_GP, O.G_FP64, O.G_LD])])
def test_multi_launch(F, maker, groups, how):
    oi = _campaign(F, maker(), 0x70151, groups, [0, 1, 2, 3], 400, how)
    assert (oi["outcome"] == O.SDC).any()


def test_k7_slot_reuse_many_replicas(F):
    """More replicas than K7 replica slots: each slot serves several replicas in
    turn, its overlay entries of the earlier ones tagged with older generations
    (they must read as absent)."""
    _campaign(F, P.multi_instance_chain(4), 0x70152, [O.G_GP, O.G_FP32, O.G_LD], [0, 1, 2, 3], 12000, "k5k7")


def test_campaign_hist_tol(F):
    prog = P.vector_add_f64()
    r = F.campaign(prog, 0x70153, [O.G_GP, O.G_FP64], [0, 1, 2, 3], 500, rtol=RTOL)
    g = O.Golden(prog)
    os_ = g.select(0x70153, [O.G_GP, O.G_FP64], [0, 1, 2, 3], 0, 500)
    oi = g.inject(os_, O.MODE_WARP_LOCAL, rtol=RTOL)
    assert np.array_equal(r.hist, O.histogram(os_, oi))
    assert np.array_equal(r.hist_tol, O.histogram(os_, oi, tol=True))
    assert ((r.inj["flags"] & F.FI_SDC_WITHIN_TOL) == (oi["flags"] & O.SDC_WITHIN_TOL)).all()
    assert not np.array_equal(r.hist, r.hist_tol)
