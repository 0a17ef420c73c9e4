"""K8 (fi_classify_batched): whole-program outcomes for multi-instance programs,
replica batches in lockstep over the launches, against the oracle's full mode
(the definition: re-run the whole program; C-12, C-14, C-19)
and against K7 (fi_classify) on the same K4 results."""
import numpy as np
import pytest

import oracle as O
from fi_inputs import programs as P

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    from paper_conf_dsn_0002hsvk21_b200 import fi
    return fi


def _run(F, prog, seed, groups, bfms, n, unchecked=False, k7=True, **kw):
    g = O.Golden(prog)
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    ic, cc = F.profile(gt)
    idx = F.SiteIndex(gt, ic, cc)
    sites = F.select_sites(idx, F.schedule(seed, groups, bfms), 0, n)
    os_ = g.select(seed, groups, bfms, 0, n)
    cap = F.log_capacity(gt)
    out, log = F.inject(gt, sites, n, cap)
    out7 = out.clone()
    hist = F.classify_batched(gt, sites, n, out, log, cap, unchecked=unchecked, **kw)
    hist7 = F.classify(gt, sites, n, out7, log, cap, unchecked=unchecked) if k7 else None
    gi = F.as_numpy(out, F.INJ_DTYPE, n)
    g7 = F.as_numpy(out7, F.INJ_DTYPE, n)
    oi = g.inject(os_, O.MODE_FULL | (O.UNCHECKED if unchecked else 0))
    for f in ("outcome", "flags", "fault_kind", "before", "after", "mask"):
        bad = np.flatnonzero(gi[f] != oi[f])
        assert bad.size == 0, f"{f}: replica {bad[0]} k8 {gi[bad[0]]} oracle {oi[bad[0]]} site {os_[bad[0]]}"
    assert (gi["fault_pc"][gi["fault_kind"] > 0] == oi["fault_pc"][oi["fault_kind"] > 0]).all()
    assert np.array_equal(hist.cpu().numpy().astype(np.uint64), O.histogram(os_, oi))
    if k7:                                    # K7's fixed-size overlay suits short programs only
        for f in ("outcome", "flags", "fault_kind"):
            assert (gi[f] == g7[f]).all(), f
        assert np.array_equal(hist.cpu().numpy(), hist7.cpu().numpy())
    return oi


@pytest.mark.parametrize("maker,unchecked", [(lambda: P.multi_instance_chain(5), False),
                                             (lambda: P.multi_instance_chain(6, shrink=29), False),
                                             (lambda: P.multi_instance_chain(4, n=300, block=96), True)])
def test_k8_chains(F, maker, unchecked):
    oi = _run(F, maker(), 0x7A7, [F.G_GP, F.G_LD, F.G_FP32, F.G_OTHERS], [0, 1, 2, 3], 400, unchecked)
    assert (oi["outcome"] == O.SDC).sum() > 0


@pytest.mark.parametrize("unchecked", [False, True])
def test_k8_scatter_wild_stores(F, unchecked):
    """Data-dependent store addresses: corrupted indices store into other warps'
    words and other buffers (C-14 order), or fault in later launches."""
    oi = _run(F, P.scatter_chain(), 7, [F.G_GP, F.G_LD], [0, 1, 2, 3], 400, unchecked)
    if unchecked:                                   # memory faults only end warps: potential DUE (f4)
        assert (oi["flags"] & O.POTENTIAL_DUE).any() and len(np.unique(oi["outcome"])) == 2
    else:
        assert len(np.unique(oi["outcome"])) == 3


def test_k8_small_batches_and_pool(F):
    """Several batches of 7 replicas; a small pool."""
    _run(F, P.scatter_chain(5, n=200, block=32, seed=3), 11, [F.G_GP], [0, 3], 120, batch=7, pool_pages=256)


def test_k8_c3_mini(F):
    oi = _run(F, P.c3(full=False), P.CAMPAIGN_SEED[3], [F.G_GP, F.G_FP64, F.G_PR, F.G_LD], [0, 1, 2, 3], 300)
    assert len(np.unique(oi["outcome"])) >= 2


def test_k8_pool_exhaustion_is_reported(F):
    prog = P.multi_instance_chain(5)
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    ic, cc = F.profile(gt)
    idx = F.SiteIndex(gt, ic, cc)
    n = 64
    sites = F.select_sites(idx, F.schedule(5, [F.G_FP32], [0]), 0, n)
    cap = F.log_capacity(gt)
    out, log = F.inject(gt, sites, n, cap)
    with pytest.raises(F.FIError) as e:
        F.classify_batched(gt, sites, n, out, log, cap, pool_pages=1)
    assert e.value.code == F.FI_E_CAPACITY
    gi = F.as_numpy(out, F.INJ_DTYPE, n)
    assert (gi["outcome"] == 0xFF).any()


def test_k8_c4_mini(F):
    """mini-C4 (ResNet-50 v1.5 shape, width 8, 32x32: 72 launches, 53 convolutions):
    trace and whole-program outcomes (K8) against the oracle."""
    from fi_inputs import resnet as R
    prog = R.c4(full=False)
    g = O.Golden(prog)
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    assert np.array_equal(F.as_numpy(gt.rec, F.RECORD_DTYPE, gt.n_rec), g.trace())
    assert np.array_equal(gt.image.cpu().numpy(), g.final_image())
    oi = _run(F, prog, R.C4_CAMPAIGN_SEED, [F.G_GP, F.G_FP32, F.G_LD, F.G_PR], [0, 1, 2, 3], 300, k7=False)
    assert (oi["outcome"] == O.SDC).any() and (oi["outcome"] == O.MASKED).any()


@pytest.mark.parametrize("which", range(5))
def test_k8_c5_mini(F, which):
    """mini C5 suite (stencil FP32, D3Q19 LBM FP64, LJ MD FP64 with divergent
    cutoff branches, EP FP64+int, CG): golden trace and whole-program outcomes."""
    from fi_inputs import hpc as H
    prog = H.c5(full=False)[which]
    g = O.Golden(prog)
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    assert np.array_equal(F.as_numpy(gt.rec, F.RECORD_DTYPE, gt.n_rec), g.trace())
    assert np.array_equal(gt.image.cpu().numpy(), g.final_image())
    groups = [F.G_GP, F.G_GPPR, F.G_LD, F.G_PR, F.G_FP64 if which in (1, 2, 3, 4) else F.G_FP32]
    oi = _run(F, prog, H.C5_CAMPAIGN_SEED + which, groups, [0, 1, 2, 3], 250, k7=which in (2, 3))
    assert (oi["outcome"] == O.SDC).any()
