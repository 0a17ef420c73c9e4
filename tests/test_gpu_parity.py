"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bit-exact for everything (counts, trace bytes, golden images, sites, injected
values, fault kinds, outcomes) — the whole path is integer or IEEE-exact (C-13),
so the tolerance is 0 everywhere.
"""
import numpy as np
import pytest
import torch

import oracle as O
import opcases
from fi_inputs import programs as P

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    from paper_conf_dsn_0002hsvk21_b200 import fi
    return fi


def _gpu_golden(F, prog, ckpt="auto"):
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp, ckpt_interval=ckpt)
    return dp, gt


def _trace_np(F, gt):
    return F.as_numpy(gt.rec, F.RECORD_DTYPE, gt.n_rec)


def _site_fields(a):
    names = [n for n in a.dtype.names if n != "pad"]
    return np.stack([a[n].astype(np.uint64) for n in names], axis=1), names


def _assert_sites_equal(g, o):
    ga, names = _site_fields(g)
    oa, _ = _site_fields(o)
    bad = np.argwhere(ga != oa)
    assert bad.size == 0, f"site {bad[0][0]} field {names[bad[0][1]]}: gpu {ga[bad[0][0]]} oracle {oa[bad[0][0]]}"


def test_ops_conformance(F):
    for name, rows, words, exp in opcases.cases(seed=77):
        prog = opcases.build(rows, words, name)
        dp, gt = _gpu_golden(F, prog)
        img = gt.image.cpu().numpy()
        y = prog.view(img, "Y", "<u4").reshape(-1, 8)
        assert np.array_equal(y, exp), name


@pytest.mark.parametrize("seed", range(40))
def test_fuzz_trace_and_image(F, seed):
    prog = P.fuzz_program(seed, n_ops=int(60 + seed * 7 % 140), block=[80, 64, 96, 33][seed % 4])
    g = O.Golden(prog)
    dp, gt = _gpu_golden(F, prog)
    assert gt.n_rec == g.n_records
    assert np.array_equal(gt.image.cpu().numpy(), g.final_image())
    assert np.array_equal(_trace_np(F, gt), g.trace())
    ic, cc = F.profile(gt)
    assert np.array_equal(ic.cpu().numpy().astype(np.uint64), g.counts())


@pytest.mark.parametrize("seed", [5, 6, 7])
def test_ffma_runs_special_values(F, seed):
    """The emulator's batched simple-FFMA path on NaN payloads, infinities, signed
    zeros and denormals: images, traces and injected outcomes against the oracle
    (which canonicalises NaN explicitly, C-13)."""
    prog = P.ffma_runs(seed)
    gi, oi = _campaign_parity(F, prog, seed, [F.G_FP32, F.G_GP, F.G_LD], [0, 1, 2, 3], 300, O.MODE_FULL)
    assert len(np.unique(oi["outcome"])) >= 2


def _campaign_parity(F, prog, seed, groups, bfms, n, mode, ckpt="auto", unchecked=False):
    g = O.Golden(prog)
    dp, gt = _gpu_golden(F, prog, ckpt)
    assert np.array_equal(_trace_np(F, gt), g.trace())
    assert np.array_equal(gt.image.cpu().numpy(), g.final_image())
    ic, cc = F.profile(gt)
    assert np.array_equal(ic.cpu().numpy().astype(np.uint64), g.counts())
    idx = F.SiteIndex(gt, ic, cc)
    sites = F.select_sites(idx, F.schedule(seed, groups, bfms), 0, n)
    gs = F.as_numpy(sites, F.SITE_DTYPE, n)
    os_ = g.select(seed, groups, bfms, 0, n)
    _assert_sites_equal(gs, os_)
    cap = F.log_capacity(gt)
    out, log = F.inject(gt, sites, n, cap)
    hist = F.classify(gt, sites, n, out, log, cap, unchecked=unchecked)
    gi = F.as_numpy(out, F.INJ_DTYPE, n)
    oi = g.inject(os_, mode | (O.UNCHECKED if unchecked else 0))
    assert (gi["flags"] == oi["flags"]).all()
    for f in ("before", "after", "mask", "fault_kind", "outcome"):
        bad = np.flatnonzero(gi[f] != oi[f])
        assert bad.size == 0, f"{f}: replica {bad[0]} gpu {gi[bad[0]]} oracle {oi[bad[0]]} site {os_[bad[0]]}"
    assert (gi["fault_pc"][gi["fault_kind"] > 0] == oi["fault_pc"][oi["fault_kind"] > 0]).all()
    assert np.array_equal(hist.cpu().numpy().astype(np.uint64), O.histogram(os_, oi))
    return gi, oi


def test_c1_full_parity(F):
    # C1: 100 replicas, G_GP, FLIP_SINGLE_BIT, oracle in full-program mode (the definition)
    _campaign_parity(F, P.c1(), P.CAMPAIGN_SEED[1], [F.G_GP], [0], 100, O.MODE_FULL)


def test_c1_all_models_groups(F):
    _campaign_parity(F, P.vector_add(n=1000), 0x1234, [F.G_GP, F.G_PR, F.G_LD, F.G_FP32, F.G_OTHERS, F.G_GPPR],
                     [0, 1, 2, 3], 600, O.MODE_FULL)


def test_mini_c2_parity(F):
    gi, oi = _campaign_parity(F, P.c2(full=False), P.CAMPAIGN_SEED[2], [F.G_GP], [0, 1, 2, 3], 400, O.MODE_WARP_LOCAL)
    assert len(np.unique(oi["outcome"])) >= 2


@pytest.mark.parametrize("seed", range(8))
def test_fuzz_campaign_parity(F, seed):
    prog = P.fuzz_program(100 + seed, n_ops=100)
    # odd checkpoint intervals make replicas restart mid-divergence (seed % 3 == 0: no checkpoints)
    _campaign_parity(F, prog, 0xABC0 + seed, [F.G_GPPR, F.G_GP, F.G_PR, F.G_FP32, F.G_FP64, F.G_OTHERS][: 1 + seed % 6],
                     [0, 1, 2, 3], 300, O.MODE_FULL, ckpt=[0, 5, 13][seed % 3])


@pytest.mark.parametrize("maker,mode", [(P.c1, O.MODE_FULL), (lambda: P.vector_add(n=1000), O.MODE_FULL),
                                        (lambda: P.c2(full=False), O.MODE_WARP_LOCAL),
                                        (lambda: P.fuzz_program(7, n_ops=90), O.MODE_FULL)])
def test_unchecked_potential_due_parity(F, maker, mode):
    """Row f4: potential-DUE semantics (FI_UNCHECKED) — outcome, flags and fault kinds match the oracle."""
    gi, oi = _campaign_parity(F, maker(), 0xF4, [F.G_GP, F.G_OTHERS], [0, 1, 2, 3], 400, mode, unchecked=True)
    assert not (gi["outcome"][gi["flags"] == 1] == F.DUE).any()


def test_mini_c2_parity_checkpoints(F):
    _campaign_parity(F, P.c2(full=False), 0x77, [F.G_GP, F.G_LD, F.G_PR], [0, 1, 2, 3], 300, O.MODE_WARP_LOCAL,
                     ckpt=97)


def test_checkpoints_do_not_change_results(F):
    prog = P.c2(full=False)
    res = []
    for ck in (0, 64, 1000, "auto"):
        dp, gt = _gpu_golden(F, prog, ck)
        ic, cc = F.profile(gt)
        idx = F.SiteIndex(gt, ic, cc)
        sites = F.select_sites(idx, F.schedule(3, [F.G_GP], [0, 1, 2, 3]), 0, 500)
        cap = F.log_capacity(gt)
        out, log = F.inject(gt, sites, 500, cap)
        F.classify(gt, sites, 500, out, log, cap)
        res.append(F.as_numpy(out, F.INJ_DTYPE, 500))
        assert np.array_equal(_trace_np(F, gt), _trace_np(F, _gpu_golden(F, prog, 0)[1]))
    for r in res[1:]:
        assert (r == res[0]).all()


def test_multi_instance_profile_and_select(F):
    prog = P.multi_instance_chain(n_inst=4)
    g = O.Golden(prog)
    dp, gt = _gpu_golden(F, prog)
    assert np.array_equal(_trace_np(F, gt), g.trace())
    ic, cc = F.profile(gt)
    assert np.array_equal(ic.cpu().numpy().astype(np.uint64), g.counts())
    idx = F.SiteIndex(gt, ic, cc)
    sites = F.select_sites(idx, F.schedule(99, [F.G_GP, F.G_LD], [0, 3]), 0, 200)
    _assert_sites_equal(F.as_numpy(sites, F.SITE_DTYPE, 200), g.select(99, [F.G_GP, F.G_LD], [0, 3], 0, 200))


def test_profile_shards_sum(F):
    prog = P.c2(full=False)
    dp, gt = _gpu_golden(F, prog)
    full, cfull = F.profile(gt)
    cut = (gt.n_rec // 3) // F.FI_CHUNK * F.FI_CHUNK
    a, ca = F.profile(gt, 0, cut)
    b, cb = F.profile(gt, cut, gt.n_rec)
    assert torch.equal(a + b, full)
    nc = cut // F.FI_CHUNK
    assert torch.equal(ca[:nc], cfull[:nc]) and torch.equal(cb[nc:], cfull[nc:])


def test_invariant_violation_detected(F):
    prog = P.c1()
    dp, gt = _gpu_golden(F, prog)
    ic, cc = F.profile(gt)
    F.SiteIndex(gt, ic, cc)                      # consistent counts pass
    bad = ic.clone()
    bad[0, F.G_GP] += 1
    with pytest.raises(F.FIError) as e:
        F.SiteIndex(gt, bad, cc)
    assert e.value.code == F.FI_E_INVARIANT
    badc = cc.clone()
    badc[0, F.G_GPPR] -= 1
    with pytest.raises(F.FIError) as e:
        F.SiteIndex(gt, ic, badc)
    assert e.value.code == F.FI_E_INVARIANT


def test_errors(F):
    prog = P.c1()
    dp, gt = _gpu_golden(F, prog)
    ic, cc = F.profile(gt)
    idx = F.SiteIndex(gt, ic, cc)
    with pytest.raises(F.FIError) as e:
        F.select_sites(idx, F.schedule(1, [F.G_NODEST], [0]), 0, 4)
    assert e.value.code == F.FI_E_NOT_INJECTABLE
    with pytest.raises(F.FIError) as e:
        F.select_sites(idx, F.schedule(1, [F.G_FP64], [0]), 0, 4)
    assert e.value.code == F.FI_E_EMPTY_GROUP
    s = F.select_sites(idx, F.schedule(1, [F.G_GP], [0]), 0, 1)
    txt = F.write_params_txt(F.as_numpy(s, F.SITE_DTYPE, 1)[0], "vecadd")
    lines = txt.strip().split("\n")
    assert len(lines) == 7 and lines[0] == str(F.G_GP) and lines[2] == "vecadd"


def test_empty_and_ragged(F):
    # ragged: n not a multiple of the block, partial warps (block = 48)
    prog = P.vector_add(n=777, grid=17, block=48)
    _campaign_parity(F, prog, 5, [F.G_GP], [0, 3], 150, O.MODE_FULL)
    # zero replicas is a no-op
    dp, gt = _gpu_golden(F, prog)
    ic, cc = F.profile(gt)
    idx = F.SiteIndex(gt, ic, cc)
    F.select_sites(idx, F.schedule(1, [F.G_GP], [0]), 0, 0)


@pytest.mark.parametrize("n", [0, 1, 255, 256, 4096, 4097, 300001, 2_500_000])
def test_scan_u64_and_rows(F, n):
    """K2 scans (decoupled lookback) against numpy cumsum: width-1 u64 and width-8
    u32 rows (the chunk index), many tiles and a ragged tail."""
    rng = np.random.Generator(np.random.PCG64(n))
    x = rng.integers(0, 2**40, n, dtype=np.uint64)
    got = F.scan_u64(torch.from_numpy(x.view(np.int64)).cuda()).cpu().numpy().view(np.uint64)
    want = np.concatenate([[0], np.cumsum(x, dtype=np.uint64)])
    assert np.array_equal(got, want)
    # width-8 u32 rows through the site index
    cc = rng.integers(0, 32768, (max(n, 1), 8), dtype=np.int64).astype(np.int32)
    ic = rng.integers(0, 2**40, (3, 8), dtype=np.int64)
    L = F.lib()
    import ctypes as C
    nb = L.fi_site_index_bytes(3, n)
    buf = torch.empty(nb, dtype=torch.uint8, device="cuda")
    cct = torch.from_numpy(cc).cuda()
    ict = torch.from_numpy(ic).cuda()
    st = F.DeviceStatus("cuda")
    rc = L.fi_build_site_index(ict.data_ptr(), 3, cct.data_ptr(), n, buf.data_ptr(), st.ptr,
                               torch.cuda.current_stream().cuda_stream)
    assert rc == 0
    torch.cuda.synchronize()
    assert int(st.t.item()) == 1 << F.FI_E_INVARIANT        # random rows violate the Table II identities
    torch.cuda.synchronize()
    b = buf.cpu().numpy()
    pk = b[: 4 * 64].view(np.uint64).reshape(4, 8)
    assert np.array_equal(pk, np.concatenate([np.zeros((1, 8), np.uint64), np.cumsum(ic.astype(np.uint64), 0)]))
    off = (4 * 64 + 255) // 256 * 256
    T = (n + 63) // 64
    pt = b[off: off + (T + 1) * 64].view(np.uint64).reshape(T + 1, 8)
    tiles = np.zeros((T, 8), np.uint64)
    for t in range(T):
        tiles[t] = cc[t * 64: min(n, t * 64 + 64)].astype(np.uint64).sum(0)
    wantt = np.concatenate([np.zeros((1, 8), np.uint64), np.cumsum(tiles, 0)])
    assert np.array_equal(pt, wantt)


@pytest.mark.parametrize("maker", [P.c1, lambda: P.fuzz_program(3), lambda: P.multi_instance_chain(4, shrink=30),
                                   lambda: P.c2(full=False)])
def test_opcode_profile_parity(F, maker):
    """Row f1: per-opcode profile equals the oracle's per-record sums, and
    sharded profiles add up."""
    prog = maker()
    g = O.Golden(prog)
    dp, gt = _gpu_golden(F, prog)
    oc = F.profile_opcodes(gt).cpu().numpy().astype(np.uint64)[: len(prog.instances)]
    assert np.array_equal(oc, g.opcode_counts())
    cut = gt.n_rec // 2 + 7
    a = F.profile_opcodes(gt, 0, cut) + F.profile_opcodes(gt, cut, gt.n_rec)
    assert np.array_equal(a.cpu().numpy().astype(np.uint64)[: len(prog.instances)], oc)


def test_approximate_profile_and_selection_parity(F):
    """Row f1: approximate profiling and selection over it, including
    the not-injected sites of C-17, bit-exact against the oracle; injection and
    classification skip not-injected sites."""
    prog = P.multi_instance_chain(n_inst=6, n=256, shrink=33)
    g = O.Golden(prog)
    dp, gt = _gpu_golden(F, prog)
    ap = F.profile_approx(gt).cpu().numpy().astype(np.uint64)
    assert np.array_equal(ap, g.approx_counts())
    idx = F.InstanceIndex(gt, F.profile_approx(gt))
    n = 500
    sched = F.schedule(0xA11, [F.G_GP, F.G_FP32, F.G_LD], [0, 1, 2, 3])
    sites = F.select_sites_approx(idx, sched, 0, n)
    gs = F.as_numpy(sites, F.SITE_DTYPE, n)
    os_ = g.select_approx(0xA11, [F.G_GP, F.G_FP32, F.G_LD], [0, 1, 2, 3], 0, n)
    _assert_sites_equal(gs, os_)
    assert 0 < (gs["flags"] == 1).sum() < n
    cap = F.log_capacity(gt)
    out, log = F.inject(gt, sites, n, cap)
    hist = F.classify(gt, sites, n, out, log, cap)
    gi = F.as_numpy(out, F.INJ_DTYPE, n)
    oi = g.inject(os_, O.MODE_FULL)
    assert (gi["outcome"] == oi["outcome"]).all()
    ok = gs["flags"] == 0
    for f in ("before", "after", "mask", "fault_kind"):
        assert (gi[f][ok] == oi[f][ok]).all(), f
    assert int(hist.sum()) == int(ok.sum())


@pytest.mark.parametrize("maker,unchecked", [(lambda: P.multi_instance_chain(5), False),
                                             (lambda: P.multi_instance_chain(6, shrink=29), False),
                                             (lambda: P.multi_instance_chain(4, n=300, block=96), True)])
def test_multi_instance_injection_parity(F, maker, unchecked):
    """K7: faults in non-final instances propagate through the later launches; the
    outcome is the whole program's (oracle full mode, the definition)."""
    gi, oi = _campaign_parity(F, maker(), 0x7A7, [F.G_GP, F.G_LD, F.G_FP32, F.G_OTHERS], [0, 1, 2, 3], 400,
                              O.MODE_FULL, unchecked=unchecked)
    assert (oi["outcome"] == O.SDC).sum() > 0


def test_c3_mini_campaign_parity(F):
    """mini-C3 (62 instances, 12 static kernels, SHFL reductions, divergent loops,
    boundary predication): trace, counts, sites and whole-program outcomes (K7)
    bit-exact against the oracle's full-program mode."""
    gi, oi = _campaign_parity(F, P.c3(full=False), P.CAMPAIGN_SEED[3], [F.G_GP, F.G_FP64, F.G_PR, F.G_LD],
                              [0, 1, 2, 3], 300, O.MODE_FULL)
    assert len(np.unique(oi["outcome"])) >= 2


def test_c3_mini_approximate(F):
    prog = P.c3(full=False)
    g = O.Golden(prog)
    dp, gt = _gpu_golden(F, prog)
    ap = F.profile_approx(gt).cpu().numpy().astype(np.uint64)
    assert np.array_equal(ap, g.approx_counts())
    assert np.array_equal(ap, g.counts())          # no data-dependent control flow in CG kernels
