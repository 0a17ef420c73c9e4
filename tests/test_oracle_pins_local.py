"""Pins for the oracle's full-size checker path: the functions the
full-size GPU parity tests use as their reference — selection without a kept
trace, ``build_site`` / ``warp_site_at`` / ``warp_site_rank``, ``inject_local``,
``count_warps`` — and a transient fault propagating through later launches.

What fixes each expected value:
  * selection: the trace-walking enumeration, itself pinned by brute force
    (``test_oracle_pins.py::test_selection_bijection``), "random
    number n from the set 1..N" in the canonical order C-3;
  * warp-local injection: ``inject(MODE_FULL)`` — the definition, re-running the
    whole program (PAPER.md:72 step (4), :206) — and numpy f32 sums on C1;
  * counts: the hand-derived closed form of the SGEMM listing (tests/closed_forms.py);
  * propagation: the chain recurrence y_{i+1} = fma(y_i, 0.5, x) evaluated by
    numpy with the corrupted word (the outcome is the whole
    program's output).
"""
import numpy as np
import pytest

import oracle as O
from closed_forms import sgemm_closed_form, sgemm_per_thread, GP, FP32
from fi_inputs import programs as P

FIELDS_SITE = [n for n in O.SITE_DTYPE.names]
FIELDS_INJ = ("before", "after", "mask", "fault_kind", "fault_pc", "outcome", "flags", "n_faulty_stores")


@pytest.fixture(scope="module")
def c1():
    return O.Golden(P.c1())


@pytest.fixture(scope="module")
def mini_c2():
    prog = P.c2(full=False)
    return prog, O.Golden(prog), O.Golden(prog, keep_trace=False)


# ---------------------------------------------------------------------------
# Selection without a kept trace (the full-size C2 checker) == enumeration
# ---------------------------------------------------------------------------
def test_c1_every_gp_site_located_without_trace(c1):
    """Every one of C1's 14,336 G_GP sites: the per-warp-count + warp re-run path
    returns the same (warp, step, lane, pc, thread, slot) as the trace walk, and
    warp_site_at / warp_site_rank invert each other on it."""
    g_nt = O.Golden(P.c1(), keep_trace=False)
    n = int(c1.counts()[0, GP])
    assert n == 14336
    s = np.arange(n, dtype=np.uint64)
    a, b = c1.locate(GP, s), g_nt.locate(GP, s)
    assert (a == b).all()
    per_warp = n // 32                                   # C1: 32 full warps, 14 GP insns per thread
    for j in range(0, n, 97):
        w, r = divmod(j, per_warp)
        st, ln, pc = O.warp_site_at(c1.prog, w, GP, r)
        assert (st, ln, pc) == (int(a["step"][j]), int(a["lane"][j]), int(a["pc"][j])) and w == int(a["warp"][j])
        assert O.warp_site_rank(c1.prog, w, GP, st, ln) == (r, per_warp)
    assert O.warp_site_at(c1.prog, 0, GP, per_warp) is None           # rank past the warp's count
    assert O.warp_site_rank(c1.prog, 0, GP, 6, 0) is None             # @P0 EXIT: not a G_GP site


def test_mini_c2_select_without_trace_and_build_site(mini_c2):
    """300 replicas of a C2-shaped campaign (G_GP, bfm = j mod 4) on mini-C2:
    select() with and without the kept trace and build_site() (draw -> warp by
    the closed-form per-warp count -> enumeration inside the warp) agree on
    every site field."""
    prog, g, g_nt = mini_c2
    seed = P.CAMPAIGN_SEED[2]
    want = g.select(seed, [GP], [0, 1, 2, 3], 0, 300)
    assert (g_nt.select(seed, [GP], [0, 1, 2, 3], 0, 300) == want).all()
    N = sgemm_closed_form(256, 256, 256)[0][GP]
    per_warp = 32 * sgemm_per_thread(256)[GP]
    assert int(g.counts()[0, GP]) == N
    rows = np.concatenate([O.build_site(prog, seed, j, GP, j % 4, per_warp, N) for j in range(300)])
    for f in FIELDS_SITE:
        assert (rows[f] == want[f]).all(), f


# ---------------------------------------------------------------------------
# inject_local (no golden handle) == inject(WARP_LOCAL) == inject(FULL)
# ---------------------------------------------------------------------------
def test_mini_c2_inject_local_equals_warp_local_and_full(mini_c2):
    prog, g, _ = mini_c2
    sites = g.select(P.CAMPAIGN_SEED[2], [GP], [0, 1, 2, 3], 0, 300)
    wl = g.inject(sites, O.MODE_WARP_LOCAL)
    loc, decided = O.inject_local(prog, sites)
    assert decided.all()                                 # no wild store outside the warp's own words here
    for f in FIELDS_INJ:
        assert (loc[f] == wl[f]).all(), f
    full = g.inject(sites[:48], O.MODE_FULL)             # the definition: whole program re-run
    for f in FIELDS_INJ:
        assert (full[f] == wl[:48][f]).all(), f
    assert set(np.unique(wl["outcome"]).tolist()) >= {1, 2}


def test_c1_inject_local_all_gp_sites(c1):
    """Every C1 G_GP site under all four bit-flip models: inject_local ==
    inject(WARP_LOCAL); a stride of them == inject(FULL)."""
    n = int(c1.counts()[0, GP])
    base = c1.locate(GP, np.arange(n, dtype=np.uint64))
    rng = np.random.Generator(np.random.PCG64(11))
    sites = base.copy()
    sites["bfm"] = np.arange(n) % 4
    ub = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
    sites["u_bit"] = ub
    sites["mask"] = [O.mask(int(b), int(u)) for b, u in zip(sites["bfm"], ub)]
    wl = c1.inject(sites, O.MODE_WARP_LOCAL)
    loc, decided = O.inject_local(c1.prog, sites)
    assert decided.all()
    for f in FIELDS_INJ:
        assert (loc[f] == wl[f]).all(), f
    full = c1.inject(sites[::23], O.MODE_FULL)
    assert (full == wl[::23]).all()
    assert set(np.unique(wl["outcome"]).tolist()) == {0, 1, 2}


# ---------------------------------------------------------------------------
# count_warps (bounded CPU baseline, reference arm) == closed form
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("w0,w1", [(0, 3), (4090, 4096), (8189, 8192)])
def test_count_warps_full_c2_closed_form(w0, w1):
    prog = P.c2(full=True)
    n, c = O.count_warps(prog, w0, w1)
    per = sgemm_per_thread(4096)
    assert c.tolist() == [32 * (w1 - w0) * x for x in per]
    assert n == (w1 - w0) * (17 + 73 * 4096 + 29)


def test_count_warps_mini_c2_whole_program(mini_c2):
    prog, g, _ = mini_c2
    want, nrec = sgemm_closed_form(256, 256, 256)
    n, c = O.count_warps(prog, 0, g.n_warps)
    assert c.tolist() == want and n == nrec
    assert (c == g.counts()[0]).all()
    n2, c2 = O.count_warps(prog, 5, 9)
    assert (c2 == g.warp_counts()[5:9].sum(0)).all() and n2 == int(g.warp_len()[5:9].sum())


# ---------------------------------------------------------------------------
# A transient fault propagating through later launches (C-19)
# ---------------------------------------------------------------------------
def _fma_chain(y, x, mask_at=None):
    """One launch of y <- fma(y, 0.5, x) in f32, NaN canonicalised (C-13).
    mask_at = (t, mask) XORs the result word of thread t.  Evaluating in f64 and
    rounding once to f32 equals the fused f32 FMA: y*0.5 is exact in f64, and the
    f64 sum of two f32 values is exact when their exponents differ by <= 29;
    otherwise the smaller one lies below 2^-29 of the larger, far from an f32
    rounding midpoint (2^-24), so the f64 rounding cannot create a tie."""
    with np.errstate(all="ignore"):
        r = (y.astype(np.float64) * 0.5 + x.astype(np.float64)).astype(np.float32)
    u = r.view("<u4").copy()
    u[np.isnan(r)] = 0x7FFFFFFF
    if mask_at is not None:
        u[mask_at[0]] ^= np.uint32(mask_at[1])
    return u.view("<f4")


@pytest.mark.parametrize("launch", [0, 1, 2, 3])
def test_transient_fault_propagates_through_later_launches(launch):
    n_inst, n = 4, 256
    prog = P.multi_instance_chain(n_inst=n_inst, n=n, block=64)
    g = O.Golden(prog)
    gold = g.final_image()
    x = prog.view(gold, "x", "<f4")
    per_launch = int(g.counts()[0, FP32])
    assert per_launch == n and (g.counts()[:, FP32] == n).all()
    rng = np.random.Generator(np.random.PCG64(100 + launch))
    ss = rng.choice(per_launch, 12, replace=False) + launch * per_launch
    outcomes = []
    for s in ss:
        site = g.locate(FP32, np.array([s], dtype=np.uint64))
        assert int(site["instance"][0]) == launch and int(site["pc"][0]) == 16      # the FFMA
        for bit in (0, 13, 23, 30, 31):
            site["mask"], site["bfm"] = 1 << bit, 0
            kind, img = g.inject_image(site)
            assert kind == 0
            t = int(site["thread"][0])
            y = prog.view(gold, "y0", "<f4")
            for i in range(n_inst):
                y = _fma_chain(y, x, (t, 1 << bit) if i == launch else None)
                assert np.array_equal(prog.view(img, f"y{i + 1}", "<u4"), y.view("<u4")), (s, bit, i)
            sdc = not np.array_equal(y.view("<u4"), prog.view(gold, f"y{n_inst}", "<u4"))
            r = g.inject(site, O.MODE_FULL)[0]
            assert r["outcome"] == (O.SDC if sdc else O.MASKED) and r["fault_kind"] == 0
            outcomes.append(int(r["outcome"]))
    if launch < n_inst - 1:
        assert O.MASKED in outcomes                      # low bits absorbed by a later launch's rounding
    assert O.SDC in outcomes


def test_transient_address_fault_in_middle_launch_is_due():
    """A flip of the high address word of the store pointer in launch 1: the
    whole program stops with an unmapped store (C-9) — DUE, and the later
    launches never run (their buffers stay zero in the faulty image)."""
    prog = P.multi_instance_chain(n_inst=4, n=256, block=64)
    g = O.Golden(prog)
    gp_per_launch = int(g.counts()[0, GP])
    # the IMAD.WIDE R10 at pc 12 is the store address pair: its G_GP site in launch 1, lane 5
    sites = g.locate(GP, np.arange(gp_per_launch, 2 * gp_per_launch, dtype=np.uint64))
    pick = np.flatnonzero((sites["pc"] == 12) & (sites["lane"] == 5) & (sites["dst_reg"] == 10))
    site = sites[pick[:1]].copy()
    assert len(site) == 1 and int(site["instance"][0]) == 1
    site["dst_reg"], site["mask"] = 11, 1 << 20
    kind, img = g.inject_image(site)
    assert kind == 2
    for i in (2, 3, 4):
        assert not prog.view(img, f"y{i}", "<u4").any()
    r = g.inject(site, O.MODE_FULL)[0]
    assert r["outcome"] == O.DUE and r["fault_kind"] == 2 and r["fault_pc"] == 17


# ---------------------------------------------------------------------------
# scan_trace (the K1 CPU baseline over a trace in host RAM)
# ---------------------------------------------------------------------------
def test_scan_trace_equals_counts_and_closed_form(mini_c2, c1):
    """The per-record sum over the kept trace equals the interpreter's counts, the
    C1 worked example and the mini-C2 closed form (Table II)."""
    prog, g, _ = mini_c2
    want, _ = sgemm_closed_form(256, 256, 256)
    assert O.scan_trace(g.trace(), 1)[0].tolist() == want
    assert O.scan_trace(c1.trace(), 1, n_threads=3)[0].tolist() == [0, 1024, 6144, 1024, 2048, 7168, 15360, 14336]
    chain = O.Golden(P.multi_instance_chain(n_inst=3, shrink=20))
    assert (O.scan_trace(chain.trace(), 3, n_threads=5) == chain.counts()).all()
    assert (O.scan_trace(chain.trace()[:0], 3) == 0).all()
