"""Pin the CPU oracle to things other than itself.

Each test names what fixes the expected value: a PAPER.md passage with a
closed form, a published known-answer vector, exact rational arithmetic,
numpy, or brute force on a tiny input.
"""
from fractions import Fraction

import numpy as np
import pytest

import oracle as O
from fi_inputs import isa, programs as P
from closed_forms import sgemm_closed_form


# ---------------------------------------------------------------------------
# RNG: Philox4x32-10 known-answer vectors (Random123 kat_vectors) and Lemire
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("ctr,key,want", [
    ([0, 0, 0, 0], [0, 0], [0x6627e8d5, 0xe169c58d, 0xbc57ac4c, 0x9b00dbd8]),
    ([0xffffffff] * 4, [0xffffffff] * 2, [0x408f276d, 0x41c83b0e, 0xa20bc7c6, 0x6d5451fd]),
    ([0x243f6a88, 0x85a308d3, 0x13198a2e, 0x03707344], [0xa4093822, 0x299f31d0],
     [0xd16cfe09, 0x94fdcceb, 0x5001e420, 0x24126ea1]),
])
def test_philox_kat(ctr, key, want):
    assert O.philox4x32_10(ctr, key) == want


def test_lemire_power_of_two_is_top_bits():
    # N = 2^k never rejects ((2^64 - N) mod N = 0) and s = x >> (64 - k) exactly.
    for j in range(200):
        for k in (1, 7, 33, 63):
            s, ud, ub, att = O.draw(0xC0FFEE, j, 1 << k)
            w = O.philox4x32_10([j & 0xFFFFFFFF, j >> 32, 0, 0x46490001], [0xC0FFEE, 0])
            x = w[0] | (w[1] << 32)
            assert att == 1 and s == x >> (64 - k) and ud == w[2] and ub == w[3]


def test_lemire_rejection_rate_and_range():
    # N = 2^63 + 1: threshold t = 2^63 - 1, so about half the first draws are rejected
    n = (1 << 63) + 1
    atts = [O.draw(7, j, n)[3] for j in range(2000)]
    assert all(O.draw(7, j, n)[0] < n for j in range(200))
    frac_retry = np.mean(np.array(atts) > 1)
    assert 0.45 < frac_retry < 0.55
    assert O.draw(1, 5, 1)[0] == 0


def test_draw_uniform_chi2():
    # PAPER.md:78 "uniform distribution": chi-square over 17 bins, 34k draws
    n, bins = 17, np.zeros(17)
    for j in range(34000):
        bins[O.draw(0xC0000001, j, n)[0]] += 1
    chi2 = ((bins - 2000) ** 2 / 2000).sum()
    assert chi2 < 39.25          # p = 0.001 critical value, 16 dof


# ---------------------------------------------------------------------------
# Table II masks against exact rationals, value = u / 2^32
# ---------------------------------------------------------------------------
EDGE_U = [0, 1, 2**27 - 1, 2**27, 2**31, 2**32 - 1, 0x80000001, 0xF8000000, 0xF7FFFFFF, 138547332, 138547333]


def _exact_masks(u):
    v = Fraction(u, 2**32)
    return [1 << int(32 * v), 3 << int(31 * v), int(0xFFFFFFFF * v)]   # int() = floor for v >= 0


def test_masks_exact():
    rng = np.random.Generator(np.random.PCG64(3))
    us = EDGE_U + [int(x) for x in rng.integers(0, 2**32, 20000)]
    for u in us:
        want = _exact_masks(u)
        got = [O.mask(b, u) for b in range(3)]
        assert got == want, (u, got, want)
        assert bin(got[0]).count("1") == 1 and got[0] < 2**32
        m2 = got[1]
        assert bin(m2).count("1") == 2 and m2 < 2**32 and (m2 & (m2 >> 1))       # two adjacent bits
    assert O.mask(3, 12345) == 0                                                 # ZERO: resolved at inject


# ---------------------------------------------------------------------------
# Table II groups with reading C-2 / slots C-6
# ---------------------------------------------------------------------------
FP64, FP32, LD, PR, NODEST, OTHERS, GPPR, GP = range(8)


def _gm(*bits):
    return sum(1 << b for b in bits)


@pytest.mark.parametrize("row,groups,gp_slots,pr_slots", [
    (isa.insn(isa.FADD, d0=3, a=1, b=2), _gm(FP32, GPPR, GP), [3], []),
    (isa.insn(isa.FFMA, d0=3, a=1, b=2, c=4), _gm(FP32, GPPR, GP), [3], []),
    (isa.insn(isa.FMNMX, d0=3), _gm(FP32, GPPR, GP), [3], []),
    (isa.insn(isa.DFMA, d0=4), _gm(FP64, GPPR, GP), [4, 5], []),
    (isa.insn(isa.FSETP, d0=2), _gm(PR, GPPR), [], [2]),             # FP32 op, predicate only -> PR
    (isa.insn(isa.DSETP, d0=1), _gm(PR, GPPR), [], [1]),
    (isa.insn(isa.ISETP, d0=isa.PT), _gm(NODEST), [], []),          # writes PT only -> no destination
    (isa.insn(isa.LDG, d0=8, mod=isa.W128), _gm(LD, GPPR, GP), [8, 9, 10, 11], []),
    (isa.insn(isa.LDG, d0=isa.RZ), _gm(NODEST), [], []),             # load into RZ
    (isa.insn(isa.LDC, d0=6, mod=isa.MOD_LDC64), _gm(LD, GPPR, GP), [6, 7], []),
    (isa.insn(isa.STG, a=4, b=8), _gm(NODEST), [], []),
    (isa.insn(isa.BRA), _gm(NODEST), [], []),
    (isa.insn(isa.EXIT), _gm(NODEST), [], []),
    (isa.insn(isa.NOP), _gm(NODEST), [], []),
    (isa.insn(isa.IADD3, d0=5, d1=2), _gm(OTHERS, GPPR, GP), [5], [2]),   # GP + PR writer
    (isa.insn(isa.IADD3, d0=5), _gm(OTHERS, GPPR, GP), [5], []),
    (isa.insn(isa.IMAD_WIDE, d0=10), _gm(OTHERS, GPPR, GP), [10, 11], []),
    (isa.insn(isa.F2F_F64_F32, d0=2), _gm(OTHERS, GPPR, GP), [2, 3], []),
    (isa.insn(isa.SHFL, d0=1), _gm(OTHERS, GPPR, GP), [1], []),
    (isa.insn(isa.MOV, d0=isa.RZ), _gm(NODEST), [], []),
])
def test_group_table(row, groups, gp_slots, pr_slots):
    r = np.array([row], dtype=isa.INSN_DTYPE)
    assert O.group_mask(r) == groups
    for g in range(8):
        if not (groups >> g) & 1 or g == NODEST:
            continue
        want = ([(1, p) for p in pr_slots] if g == PR else
                [(0, x) for x in gp_slots] + ([(1, p) for p in pr_slots] if g == GPPR else []))
        assert O.dest_slots(r, g) == want
    assert O.dest_slots(r, NODEST) == []


def _invariants(counts):
    c = counts.astype(np.int64)
    assert (c[:, GP] == c[:, FP64] + c[:, FP32] + c[:, LD] + c[:, OTHERS]).all()
    assert (c[:, GPPR] == c[:, GP] + c[:, PR]).all()
    # total = GPPR + NODEST; the six base groups partition all instructions
    assert (c[:, GPPR] + c[:, NODEST] == c[:, [FP64, FP32, LD, PR, NODEST, OTHERS]].sum(1)).all()


# ---------------------------------------------------------------------------
# Counting — closed forms
# ---------------------------------------------------------------------------
def test_c1_worked_example():
    g = O.Golden(P.c1())
    c = g.counts()
    # SURVEY §8(c) / DESIGN.md §5: per thread OTHERS 7, LD 6, PR 1, FP32 1, NODEST 2,
    # the @P0 EXIT is predicated off in every lane (n = 1024 threads) and not counted
    assert c.tolist() == [[0, 1024, 6144, 1024, 2048, 7168, 15360, 14336]]
    assert g.n_records == 576
    _invariants(c)
    t = g.trace()
    assert (t["instance"] == 0).all()
    pcs = (t["insn"] & 0xFFFF).reshape(32, 18)
    assert (pcs == np.arange(18)).all()
    assert (t["active"] == 0xFFFFFFFF).all()
    pred = t["pred"].reshape(32, 18)
    assert (pred[:, 6] == 0).all() and (np.delete(pred, 6, axis=1) == 0xFFFFFFFF).all()
    # golden output is the IEEE f32 sum (numpy)
    prog = g.prog
    img = g.final_image()
    a, b, cc = (prog.view(img, n, "<f4") for n in "abc")
    assert np.array_equal(cc.view("<u4"), (a + b).view("<u4"))


def test_predicated_off_lanes_not_counted():
    # n = 1000 < 1024 threads: 24 threads take the EXIT at pc 6 (counted, NODEST)
    g = O.Golden(P.vector_add(n=1000))
    c = g.counts()[0].tolist()
    full, cut = 1000, 24
    want = [0, full, 6 * full + cut, full + cut, 2 * full + cut, 7 * full + 4 * cut, 0, 0]
    want[GP] = want[FP32] + want[LD] + want[OTHERS]
    want[GPPR] = want[GP] + want[PR]
    assert c == want
    assert g.n_records == 576


def test_mini_c2_closed_form_and_numerics():
    prog = P.c2(full=False)
    g = O.Golden(prog, keep_trace=False)
    want, nrec = sgemm_closed_form(256, 256, 256)
    assert g.counts()[0].tolist() == want
    assert g.n_records == nrec
    _invariants(g.counts())
    # numerics: C within the FMA-chain error bound of the exact product (f64)
    img = g.final_image()
    A = prog.view(img, "A", "<f4").reshape(256, 256).astype(np.float64)    # [k][m]
    B = prog.view(img, "B", "<f4").reshape(256, 256).astype(np.float64)    # [k][n]
    C = prog.view(img, "C", "<f4").reshape(256, 256).astype(np.float64)
    exact = A.T @ B
    bound = 256 * 2.0**-24 * (np.abs(A).T @ np.abs(B)) * 1.01
    assert (np.abs(C - exact) <= bound).all()


@pytest.mark.parametrize("seed", range(6))
def test_invariants_fuzz(seed):
    g = O.Golden(P.fuzz_program(seed))
    c = g.counts()
    _invariants(c)
    t = g.trace()
    assert c.sum() > 0
    # counts <= 32 x records, and counts equal popc(active & pred) per record (brute force)
    ex = np.array([bin(int(a) & int(p)).count("1") for a, p in zip(t["active"], t["pred"])])
    gm = (t["insn"] >> 24).astype(np.int64)
    for gi in range(8):
        assert c[0, gi] == ex[(gm >> gi) & 1 == 1].sum()
        assert c[0, gi] <= 32 * len(t)


def test_multi_instance_counts():
    prog = P.multi_instance_chain(n_inst=3)
    g = O.Golden(prog)
    c = g.counts()
    _invariants(c)
    assert (c == c[0]).all()                  # identical launches -> identical counts
    assert c[0, FP32] == 256
    img = g.final_image()
    x = prog.view(img, "x", "<f4")
    y = prog.view(img, "y0", "<f4")
    for i in range(3):                        # y_{i+1} = fma(y_i, 0.5, x): exact for these values
        y = (y.astype(np.float64) * 0.5 + x.astype(np.float64)).astype(np.float32)
        assert np.array_equal(prog.view(img, f"y{i + 1}", "<f4"), y)


# ---------------------------------------------------------------------------
# Selection: brute-force bijection on tiny traces
# ---------------------------------------------------------------------------
def _enumerate_sites(trace, woff, g):
    out = []
    for w in range(len(woff) - 1):
        for r in range(woff[w], woff[w + 1]):
            rec = trace[r]
            if not (int(rec["insn"]) >> (24 + g)) & 1:
                continue
            ex = int(rec["active"]) & int(rec["pred"])
            for lane in range(32):
                if (ex >> lane) & 1:
                    out.append((w, r - woff[w], lane))
    return out


@pytest.mark.parametrize("maker", [P.c1, lambda: P.fuzz_program(11), lambda: P.multi_instance_chain(2)])
def test_selection_bijection(maker):
    prog = maker()
    g = O.Golden(prog)
    t = g.trace()
    wl = g.warp_len()
    woff = np.concatenate([[0], np.cumsum(wl)]).astype(np.int64)
    for grp in (FP32, LD, PR, OTHERS, GPPR, GP):
        sites = _enumerate_sites(t, woff, grp)
        n = int(g.counts()[:, grp].sum())
        assert len(sites) == n
        if n == 0:
            continue
        got = g.locate(grp, np.arange(n))
        assert [(int(s["warp"]), int(s["step"]), int(s["lane"])) for s in got] == sites
        # instruction_count restarts at every dynamic kernel instance
        inst_first = np.concatenate([[0], np.cumsum(g.counts()[:, grp])])
        assert (got["instruction_count"] == got["s"] - inst_first[got["instance"]]).all()


def test_select_schedule_and_slots():
    prog = P.c1()
    g = O.Golden(prog)
    s = g.select(0xC0000001, [GP, PR], [0, 1, 2, 3], 0, 64)
    assert (s["group"] == np.array([GP, PR] * 32)).all()
    assert (s["bfm"] == np.array([(j // 2) % 4 for j in range(64)])).all()
    for site in s:
        slots = O.dest_slots(prog.code[int(site["pc"])], int(site["group"]))
        assert int(site["slot"]) == (len(slots) * int(site["u_dst"])) >> 32
        assert slots[int(site["slot"])] == (int(site["dst_kind"]), int(site["dst_reg"]))
    with pytest.raises(O.OracleError):
        g.select(1, [NODEST], [0], 0, 1)                       # C-16
    with pytest.raises(O.OracleError):
        g.select(1, [FP64], [0], 0, 1)                         # empty group


# ---------------------------------------------------------------------------
# Injection + classification special cases (Table V, C-9..C-14)
# ---------------------------------------------------------------------------
def _site(g, pc, warp=0, lane=0, kind=0, reg=0, bfm=0, mask=1, group=GP):
    s = np.zeros(1, dtype=O.SITE_DTYPE)
    s["warp"], s["step"], s["pc"], s["lane"] = warp, pc, pc, lane       # C1: step == pc (no divergence)
    s["dst_kind"], s["dst_reg"], s["bfm"], s["mask"], s["group"] = kind, reg, bfm, mask, group
    s["instance"] = 0
    return s


def test_outcome_special_cases():
    g = O.Golden(P.c1())
    for mode in (O.MODE_FULL, O.MODE_WARP_LOCAL):
        # high half of the address pair (IMAD.WIDE R4 at pc 8) -> unmapped -> DUE
        r = g.inject(_site(g, 8, reg=5, mask=1 << 20), mode)[0]
        assert r["outcome"] == O.DUE and r["fault_kind"] == 2 and r["fault_pc"] == 11
        # low two address bits of the LDG.32 base -> misaligned -> DUE
        for bit in (0, 1):
            r = g.inject(_site(g, 8, reg=4, mask=1 << bit), mode)[0]
            assert r["outcome"] == O.DUE and r["fault_kind"] == 1
        # ZERO_VALUE of a zero register (R1 = ctaid = 0 in warp 0) -> Masked
        r = g.inject(_site(g, 1, reg=1, bfm=3, mask=0), mode)[0]
        assert r["before"] == 0 and r["after"] == 0 and r["outcome"] == O.MASKED
        # FLIP_SINGLE_BIT in the FADD result -> SDC
        r = g.inject(_site(g, 15, reg=8, mask=1 << 3), mode)[0]
        assert r["outcome"] == O.SDC and r["after"] == r["before"] ^ 8
        # dead register: R2 (ntid) after its last use at pc 3 is dead; inject at pc 3 into R0?
        # use the predicate written by ISETP at pc 5: flipping P0 -> EXIT taken -> store skipped -> SDC
        r = g.inject(_site(g, 5, kind=1, reg=0, group=PR), mode)[0]
        assert r["outcome"] == O.SDC and r["before"] == 0 and r["after"] == 1
        # RANDOM_VALUE on a predicate sets it to bit 31 of the mask (C-7)
        r = g.inject(_site(g, 5, kind=1, reg=0, bfm=2, mask=0x7FFFFFFF, group=PR), mode)[0]
        assert r["after"] == 0 and r["outcome"] == O.MASKED


def test_unchecked_fault_is_potential_due():
    """Row f4 [PAPER.md:208]: with unchecked errors an unmapped load only ends the
    faulting warp; its 32 outputs of c are never written (stay 0) -> SDC, flagged
    potential DUE.  A hang stays DUE."""
    prog = P.c1()
    g = O.Golden(prog)
    for mode in (O.MODE_FULL, O.MODE_WARP_LOCAL):
        r = g.inject(_site(g, 8, warp=3, reg=5, mask=1 << 20), mode | O.UNCHECKED)[0]
        assert r["outcome"] == O.SDC and r["flags"] == O.POTENTIAL_DUE and r["fault_kind"] == 2
        r = g.inject(_site(g, 8, warp=3, reg=5, mask=1 << 20), mode)[0]
        assert r["outcome"] == O.DUE and r["flags"] == 0
    hang = P.sgemm(128, 128, 4)
    gh = O.Golden(hang)
    r = gh.inject(_site(gh, 87, reg=P.KCNT, mask=1 << 30), O.MODE_FULL | O.UNCHECKED)[0]
    assert r["outcome"] == O.DUE and r["fault_kind"] == 3 and r["flags"] == 0


def test_dead_register_is_masked():
    # MOV R5 <- 7 that nothing reads, inside an otherwise C1-like kernel
    s = isa.Asm()
    s.s2r(0, isa.SR_TID)
    s.mov(5, imm=7)                       # dead
    s.ldc(2, 0, wide=True)
    s.imad_wide(2, 0, imm=4, c=2, unsigned=True)
    s.stg(2, 0)
    s.exit()
    from fi_inputs.program import ProgramBuilder, ptr_words
    pb = ProgramBuilder("dead")
    k = pb.add_kernel("dead", s.assemble())
    y = pb.add_buffer("y", 128, writer=0, output=True)
    pb.add_instance(k, 1, 32, ptr_words(y))
    g = O.Golden(pb.build())
    for mode in (O.MODE_FULL, O.MODE_WARP_LOCAL):
        for bfm, m in ((0, 1), (1, 3 << 7), (2, 0x12345678), (3, 0)):
            r = g.inject(_site(g, 1, lane=9, reg=5, bfm=bfm, mask=m), mode)[0]
            assert r["outcome"] == O.MASKED and r["before"] == 7


def test_c1_outcomes_match_numpy():
    """Every FP32/LD-result site of C1 x 32 single-bit flips: the outcome is fixed by
    the IEEE f32 sum of the corrupted operands (numpy), SDC iff the sum's bits change."""
    prog = P.c1()
    g = O.Golden(prog)
    img = g.final_image()
    a, b = prog.view(img, "a", "<f4"), prog.view(img, "b", "<f4")
    sites = []
    want = []
    for w in range(0, 32, 5):
        for lane in range(0, 32, 3):
            t = w * 32 + lane
            for pc, reg in ((11, 8), (12, 9), (15, 8)):
                for bit in range(32):
                    s = _site(g, pc, warp=w, lane=lane, reg=reg, mask=1 << bit)
                    sites.append(s)
                    av, bv = a[t:t + 1].copy(), b[t:t + 1].copy()
                    if pc == 11:
                        av = (av.view("<u4") ^ np.uint32(1 << bit)).view("<f4")
                    elif pc == 12:
                        bv = (bv.view("<u4") ^ np.uint32(1 << bit)).view("<f4")
                    with np.errstate(all="ignore"):
                        out = (av + bv).view("<u4")[0]
                    if pc == 15:
                        out = out ^ (1 << bit)
                    if np.isnan((av + bv)[0]):
                        out = 0x7FFFFFFF
                    gold = (a[t:t + 1] + b[t:t + 1]).view("<u4")[0]
                    want.append(O.SDC if out != gold else O.MASKED)
    sites = np.concatenate(sites)
    for mode in (O.MODE_FULL, O.MODE_WARP_LOCAL):
        r = g.inject(sites, mode)
        assert r["outcome"].tolist() == want


def test_full_vs_warp_local_exhaustive_c1():
    """All GP sites of warps 0 and 31, every bit, FLIP_SINGLE_BIT: the two
    classification modes (definition vs C-14 warp-local) agree outcome for outcome."""
    prog = P.vector_add(n=1000)                # warp 31 diverges at the EXIT
    g = O.Golden(prog)
    t = g.trace()
    wl = g.warp_len()
    woff = np.concatenate([[0], np.cumsum(wl)]).astype(np.int64)
    all_sites = _enumerate_sites(t, woff, GP)
    sel = [i for i, (w, st, l) in enumerate(all_sites) if w in (0, 31)][::3]
    base = g.locate(GP, np.array(sel))
    reps = []
    for s in base:
        slots = O.dest_slots(prog.code[int(s["pc"])], GP)
        for k, reg in slots:
            for bit in range(32):
                x = s.copy()
                x["dst_kind"], x["dst_reg"], x["mask"], x["bfm"] = k, reg, 1 << bit, 0
                reps.append(x)
    reps = np.array(reps, dtype=O.SITE_DTYPE)
    r1 = g.inject(reps, O.MODE_FULL)
    r2 = g.inject(reps, O.MODE_WARP_LOCAL)
    assert (r1 == r2).all()
    assert set(np.unique(r1["outcome"]).tolist()) == {0, 1, 2}


def test_watchdog_hang_is_due():
    # flip the loop counter's sign bit in mini-SGEMM: the loop runs ~2^31 times -> watchdog DUE
    prog = P.sgemm(128, 128, 4)
    g = O.Golden(prog)
    # IADD3 KCNT at pc 17 + 4 + 64 + 2 = 87 in iteration 0 (step 87)
    s = _site(g, 87, reg=P.KCNT, mask=1 << 30)
    r = g.inject(s, O.MODE_WARP_LOCAL)[0]
    assert r["outcome"] == O.DUE and r["fault_kind"] == 3
    r = g.inject(s, O.MODE_FULL)[0]
    assert r["outcome"] == O.DUE and r["fault_kind"] == 3


# ---------------------------------------------------------------------------
# PAPER.md:214 confidence margins
# ---------------------------------------------------------------------------
def test_ci_margins():
    assert round(O.ci_margin(100, 0.90), 2) == 0.08          # "+-8%"
    assert round(O.ci_margin(1000, 0.95), 2) == 0.03         # "+-3%"


# ---------------------------------------------------------------------------
# Row f1: per-opcode profile and approximate profiling
# ---------------------------------------------------------------------------
def test_c1_opcode_profile_closed_form():
    g = O.Golden(P.c1())
    oc = g.opcode_counts()[0]
    want = {isa.S2R: 3, isa.IMAD: 1, isa.LDC: 4, isa.ISETP: 1, isa.EXIT: 1, isa.IMAD_WIDE: 3, isa.LDG: 2,
            isa.FADD: 1, isa.STG: 1}           # per thread; the @P0 EXIT is predicated off
    for op in range(32):
        assert int(oc[op]) == 1024 * want.get(op, 0), isa.OPNAMES[op] if op < len(isa.OPNAMES) else op
    c = g.counts()[0]
    assert int(oc.sum()) == int(c[GPPR] + c[NODEST])


def test_approximate_profile_reuses_first_instance():
    prog = P.multi_instance_chain(n_inst=5, n=256, shrink=40)
    g = O.Golden(prog)
    exact, approx = g.counts(), g.approx_counts()
    assert (approx == exact[0]).all()                      # every instance assumed = the first
    assert (exact[1:, GP] < exact[0, GP]).all()            # later launches really are shorter
    s = g.select_approx(0xA9, [GP, FP32], [0, 1], 0, 400)
    exact_first = np.concatenate([[0], np.cumsum(exact[:, GP])]), np.concatenate([[0], np.cumsum(exact[:, FP32])])
    for site in s:
        grp = int(site["group"])
        k, ic = int(site["instance"]), int(site["instruction_count"])
        col = GP if grp == GP else FP32
        if ic >= exact[k, col]:
            assert site["flags"] == 1                      # C-17: not injected
            continue
        assert site["flags"] == 0
        # the same site as the exact enumeration's (instance-start + ic)-th
        ref = g.locate(grp, [exact_first[0 if grp == GP else 1][k] + ic])[0]
        for f in ("warp", "step", "lane", "pc", "thread"):
            assert site[f] == ref[f]
    assert 0 < (s["flags"] == 1).sum() < len(s)
    r = g.inject(s, O.MODE_FULL)
    assert (r["outcome"][s["flags"] == 1] == O.NOT_INJECTED).all()
    assert (r["outcome"][s["flags"] == 0] != O.NOT_INJECTED).all()


def test_c3_cg_numerics_and_structure():
    """mini-C3 (FP64 CG, 2-D Laplacian): the oracle's golden x equals an
    independent numpy CG of the same recurrences to 1e-12 (different summation
    order / no FMA), counts satisfy Table II per instance, and instances of one
    static kernel have identical counts (no data-dependent control flow)."""
    nx, ny, iters = 32, 16, 6
    prog = P.cg_program(nx, ny, iters)
    g = O.Golden(prog)
    img = g.final_image()
    b = prog.view(img, "b", "<f8").copy()

    def A(v):
        V = v.reshape(ny, nx)
        out = 4 * V.copy()
        out[:, 1:] -= V[:, :-1]
        out[:, :-1] -= V[:, 1:]
        out[1:, :] -= V[:-1, :]
        out[:-1, :] -= V[1:, :]
        return out.ravel()

    x, r, p = np.zeros_like(b), b.copy(), b.copy()
    rr = r @ r
    for _ in range(iters):
        ap = A(p)
        alpha = rr * (1.0 / (p @ ap))
        x = x + alpha * p
        r = r - alpha * ap
        rrn = r @ r
        beta = rrn * (1.0 / rr)
        p = r + beta * p
        rr = rrn
    xg = prog.view(img, f"x{iters}", "<f8")
    assert np.allclose(xg, x, rtol=1e-12, atol=1e-12)
    c = g.counts()
    _invariants(c)
    kern = prog.instances["kernel"]
    for k in np.unique(kern):
        rows = c[kern == k]
        assert (rows == rows[0]).all()
    assert (c[:, FP64] > 0).sum() >= 6 and len(np.unique(kern)) == 12
