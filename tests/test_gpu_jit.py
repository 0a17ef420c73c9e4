"""The JIT-specialised emulator (fi_jit_build / fi_inject_jit): per-program
generated CUDA compiled by NVRTC must give results bit-identical to the
shared-memory interpreter (fi_inject) — every fi_inj field and every logged
faulty store — and to the CPU oracle (the oracle comparisons of
test_gpu_parity.py run on the JIT path, fi.inject's default engine)."""
import numpy as np
import pytest
import torch

import oracle as O
from fi_inputs import hpc as H
from fi_inputs import programs as P
from fi_inputs import resnet as RN

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    from paper_conf_dsn_0002hsvk21_b200 import fi
    return fi


def _both(F, prog, seed, groups, bfms, n, ckpt="auto", approx=False):
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp, ckpt_interval=ckpt)
    if approx:
        idx = F.InstanceIndex(gt, F.profile_approx(gt))
        sites = F.select_sites_approx(idx, F.schedule(seed, groups, bfms), 0, n)
    else:
        ic, cc = F.profile(gt)
        sites = F.select_sites(F.SiteIndex(gt, ic, cc), F.schedule(seed, groups, bfms), 0, n)
    cap = F.log_capacity(gt)
    res = {}
    for eng in ("interp", "jit"):
        out, log = F.inject(gt, sites, n, cap, engine=eng)
        torch.cuda.synchronize()
        res[eng] = (F.as_numpy(out, F.INJ_DTYPE, n).copy(), log.view(-1, 16).cpu().numpy().copy())
    a, b = res["interp"][0], res["jit"][0]
    for f in a.dtype.names:
        bad = np.flatnonzero(a[f] != b[f])
        assert bad.size == 0, f"{f}: replica {bad[0]} interp {a[bad[0]]} jit {b[bad[0]]}"
    la, lb = res["interp"][1].reshape(n, cap, 16), res["jit"][1].reshape(n, cap, 16)
    for i in range(n):
        k = min(int(a["n_faulty_stores"][i]), cap)
        assert np.array_equal(la[i, :k], lb[i, :k]), f"faulty store log of replica {i}"
    return a, F.as_numpy(sites, F.SITE_DTYPE, n)


def test_jit_c1(F):
    a, s = _both(F, P.c1(), P.CAMPAIGN_SEED[1], [F.G_GP, F.G_PR, F.G_GPPR], [0, 1, 2, 3], 400)
    assert len(np.unique(a["outcome"] * 0 + a["fault_kind"])) >= 2


@pytest.mark.parametrize("seed", range(24))
def test_jit_fuzz(F, seed):
    prog = P.fuzz_program(300 + seed, n_ops=int(60 + seed * 11 % 140), block=[80, 64, 96, 33][seed % 4])
    _both(F, prog, 0xBEE0 + seed, [F.G_GPPR, F.G_GP, F.G_PR, F.G_FP32, F.G_FP64, F.G_OTHERS][: 1 + seed % 6],
          [0, 1, 2, 3], 300, ckpt=[0, 5, 13, "auto"][seed % 4])


def test_jit_mini_c2(F):
    a, _ = _both(F, P.c2(full=False), 0x77, [F.G_GP, F.G_LD, F.G_PR, F.G_OTHERS], [0, 1, 2, 3], 600)
    assert (a["fault_kind"] == 3).sum() + (a["fault_kind"] == 2).sum() > 0


def test_jit_job_dealing_covers_every_replica(F):
    """K4's job order (jit_prelude.cuh jnext_job): the head of the LPT list is dealt
    to the SMs in snake order, the rest comes off the shared counter, idle warps steal
    undealt rounds.  Every replica must be run exactly once whatever n is relative to
    the resident warps (dealt = min(n, grid*4)): each subset's results equal the same
    replicas' rows of one large launch, field by field, for n below, at and above
    the dealt boundary."""
    dp = F.DeviceProgram(P.c2(full=False))
    gt = F.golden_run(dp)
    ic, cc = F.profile(gt)
    N = 4000
    sites = F.select_sites(F.SiteIndex(gt, ic, cc), F.schedule(0x5151, [F.G_GP, F.G_LD], [0, 1, 2, 3]), 0, N)
    cap = F.log_capacity(gt)
    out, _ = F.inject(gt, sites, N, cap)
    ref = F.as_numpy(out, F.INJ_DTYPE, N).copy()
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    rows = sites.view(N, -1)
    for n in (1, 2, sms - 1, sms + 1, 3 * sms * 4 - 1, 3 * sms * 4, 3 * sms * 4 + 1):
        n = min(n, N)
        o2, _ = F.inject(gt, rows[:n].contiguous().view(-1), n, cap)
        torch.cuda.synchronize()
        got = F.as_numpy(o2, F.INJ_DTYPE, n)
        for f in ref.dtype.names:
            bad = np.flatnonzero(got[f] != ref[f][:n])
            assert bad.size == 0, f"n={n} {f}: replica {bad[0]}"


@pytest.mark.parametrize("seed", [5, 6, 7])
def test_jit_ffma_special_values(F, seed):
    _both(F, P.ffma_runs(seed), seed, [F.G_FP32, F.G_GP, F.G_LD], [0, 1, 2, 3], 300)


@pytest.mark.parametrize("maker", [lambda: P.multi_instance_chain(6, shrink=29), P.scatter_chain,
                                   lambda: P.c3(full=False), lambda: RN.c4(full=False)])
def test_jit_multi_launch(F, maker):
    _both(F, maker(), 0x4A11, [F.G_GP, F.G_LD, F.G_GPPR, F.G_OTHERS], [0, 1, 2, 3], 400)


def test_jit_approximate_not_injected(F):
    a, s = _both(F, P.multi_instance_chain(n_inst=6, n=256, shrink=33), 0xA11, [F.G_GP, F.G_FP32], [0, 1, 2, 3], 300,
                 approx=True)
    assert ((s["flags"] == 1) == (a["outcome"] == F.NOT_INJECTED)).all()


@pytest.mark.parametrize("which", range(5))
def test_jit_c5_minis(F, which):
    prog = H.c5(full=False)[which]
    _both(F, prog, 0xC5, [F.G_GP, F.G_GPPR, F.G_PR], [0, 1, 2, 3], 300)


def _golden_both(F, prog, ckpt):
    dp = F.DeviceProgram(prog)
    a = F.golden_run(dp, ckpt_interval=ckpt, engine="interp")
    b = F.golden_run(dp, ckpt_interval=ckpt, engine="jit")
    torch.cuda.synchronize()
    assert a.n_rec == b.n_rec and a.n_gstore == b.n_gstore
    assert torch.equal(a.warp_len, b.warp_len)
    assert torch.equal(a.image, b.image), "golden final image"
    assert torch.equal(a.rec[: a.n_rec * 16], b.rec[: b.n_rec * 16]), "trace records"
    assert torch.equal(a.gstore[: a.n_gstore * 16], b.gstore[: b.n_gstore * 16]), "golden store log"
    # the golden run's profile (fused into the JIT pass 2; K1 inside the interpreter
    # run) is K1's over the finished trace
    ic, cc = F.profile(b)
    for g in (a, b):
        gi, gc = F.golden_profile(g)
        assert torch.equal(gi, ic), "golden-run inst_counts"
        assert torch.equal(gc, cc), "golden-run chunk_counts"
    assert a.ckpt_interval == b.ckpt_interval
    if a.ckpt is not None:
        assert torch.equal(a.ckpt, b.ckpt), "register-file checkpoints"
    return a


@pytest.mark.parametrize("ckpt", [0, 5, 13, "auto"])
@pytest.mark.parametrize("maker", [P.c1, lambda: P.fuzz_program(3, n_ops=120), lambda: P.fuzz_program(8, block=33),
                                   lambda: P.c2(full=False), lambda: P.multi_instance_chain(6, shrink=29),
                                   P.scatter_chain, lambda: P.c3(full=False), lambda: P.ffma_runs(5)])
def test_jit_golden_passes(F, maker, ckpt):
    """Golden passes 1 and 2 on the JIT module: lengths, final image, trace records,
    store log, checkpoints and the run's profile byte-identical to the interpreter's."""
    _golden_both(F, maker(), ckpt)


@pytest.mark.parametrize("which", range(5))
def test_jit_golden_c5_minis(F, which):
    _golden_both(F, H.c5(full=False)[which], 7)


def _k8_both(F, prog, seed, groups, bfms, n, unchecked=False, **kw):
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    ic, cc = F.profile(gt)
    sites = F.select_sites(F.SiteIndex(gt, ic, cc), F.schedule(seed, groups, bfms), 0, n)
    cap = F.log_capacity(gt)
    out, log = F.inject(gt, sites, n, cap)
    res = {}
    for eng in ("interp", "jit"):
        o = out.clone()
        h = F.classify_batched(gt, sites, n, o, log, cap, unchecked=unchecked, engine=eng, **kw)
        torch.cuda.synchronize()
        res[eng] = (F.as_numpy(o, F.INJ_DTYPE, n).copy(), h.cpu().numpy())
    a, b = res["interp"][0], res["jit"][0]
    for f in a.dtype.names:
        bad = np.flatnonzero(a[f] != b[f])
        assert bad.size == 0, f"{f}: replica {bad[0]} interp {a[bad[0]]} jit {b[bad[0]]}"
    assert np.array_equal(res["interp"][1], res["jit"][1])
    return a


@pytest.mark.parametrize("maker,unchecked", [(lambda: P.multi_instance_chain(6, shrink=29), False),
                                             (lambda: P.multi_instance_chain(4, n=300, block=96), True),
                                             (P.scatter_chain, False), (P.scatter_chain, True),
                                             (lambda: P.c3(full=False), False), (lambda: RN.c4(full=False), False)])
def test_jit_k8(F, maker, unchecked):
    """K8's per-launch re-execution on the JIT module (fi_classify_batched_jit):
    outcomes, flags, first downstream faults and histograms identical to the
    interpreter's K8 (which test_gpu_batched.py pins to the oracle)."""
    a = _k8_both(F, maker(), 0x5A5, [F.G_GP, F.G_LD, F.G_OTHERS], [0, 1, 2, 3], 300, unchecked)
    assert (a["outcome"] == F.SDC).sum() > 0


def test_jit_k8_counts_its_steps(F):
    """fi_classify_batched_jit leaves the emulated warp-steps of every warp it
    re-executed in the workspace's first 8 bytes (fi.h; the bench's K8 roofline):
    positive when replicas propagate, and at most every replica re-running every
    warp of every launch after its faulty one (golden lengths, the watchdog aside),
    and the same count on a second identical call."""
    prog = P.multi_instance_chain(6, shrink=29)
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    ic, cc = F.profile(gt)
    n = 200
    sites = F.select_sites(F.SiteIndex(gt, ic, cc), F.schedule(0x5A5, [F.G_GP], [0]), 0, n)
    cap = F.log_capacity(gt)
    out, log = F.inject(gt, sites, n, cap)
    counts = []
    for _ in range(2):
        F.classify_batched(gt, sites, n, out.clone(), log, cap, engine="jit", steps_out=counts)
    bound = n * int(gt.warp_len.cpu().numpy().astype(np.int64).sum())
    assert 0 < counts[0] <= bound and counts[0] == counts[1], (counts, bound)


@pytest.mark.parametrize("which", range(5))
def test_jit_k8_c5_minis(F, which):
    _k8_both(F, H.c5(full=False)[which], 0xC5C5, [F.G_GP, F.G_GPPR], [0], 200, batch=64)
