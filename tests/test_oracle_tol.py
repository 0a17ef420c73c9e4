"""Pins of the oracle's C-12 secondary numeric classification (DESIGN.md §4:
rtol = 1e-6, atol = 0, NaN != number — BASELINE.md §2; the paper leaves the
SDC check to the user, "Output file is different" [PAPER.md:189], "both
application and user dependent" [PAPER.md:204]).

The expected flag comes from numpy: the faulty output element is computed by
numpy IEEE arithmetic from the corrupted operand (or the corrupted result
word), and the definition is evaluated on numpy float64 values — independent
of the oracle's interpreter and of its tolerance helper.
"""
import numpy as np
import pytest

import oracle as O
from fi_inputs import programs as P

RTOL = 1e-6
GP = O.G_GP


def _within(f: float, g: float) -> bool:
    return bool(np.isfinite(f) and np.isfinite(g) and abs(f - g) <= RTOL * abs(g))


def _site(pc, warp, lane, reg, mask, kind=0, group=GP):
    s = np.zeros(1, dtype=O.SITE_DTYPE)
    s["warp"], s["step"], s["pc"], s["lane"] = warp, pc, pc, lane        # no divergence: step == pc
    s["dst_kind"], s["dst_reg"], s["mask"], s["group"], s["bfm"] = kind, reg, mask, group, 0
    return s


def _check(g, sites, want_out, want_within):
    for mode in (O.MODE_FULL, O.MODE_WARP_LOCAL):
        r = g.inject(sites, mode, rtol=RTOL)
        assert r["outcome"].tolist() == want_out
        got = ((r["flags"] & O.SDC_WITHIN_TOL) != 0).tolist()
        assert got == want_within
        r0 = g.inject(sites, mode)                                   # rtol = 0: bitwise only, no flag
        assert (r0["outcome"] == r["outcome"]).all() and not (r0["flags"] & O.SDC_WITHIN_TOL).any()


def test_c1_f32_flips_against_numpy():
    """C1 (f32): single-bit flips of the FADD result and of both loaded operands,
    all 32 bits, for a spread of threads."""
    prog = P.c1()
    g = O.Golden(prog)
    img = g.final_image()
    a, b = prog.view(img, "a", "<f4"), prog.view(img, "b", "<f4")
    sites, out, within = [], [], []
    for w in (0, 7, 19, 31):
        for lane in (0, 13, 31):
            t = w * 32 + lane
            gold = (a[t:t + 1] + b[t:t + 1])
            for pc, reg in ((11, 8), (12, 9), (15, 8)):
                for bit in range(32):
                    av, bv = a[t:t + 1].copy(), b[t:t + 1].copy()
                    if pc == 11:
                        av = (av.view("<u4") ^ np.uint32(1 << bit)).view("<f4")
                    elif pc == 12:
                        bv = (bv.view("<u4") ^ np.uint32(1 << bit)).view("<f4")
                    with np.errstate(all="ignore"):
                        f = av + bv
                    fu = f.view("<u4")[0]
                    if pc == 15:
                        fu = fu ^ (1 << bit)
                    if np.isnan(np.array([fu], "<u4").view("<f4")[0]):
                        fu = 0x7FFFFFFF
                    gu = gold.view("<u4")[0]
                    sdc = int(fu) != int(gu)
                    fv = float(np.array([fu], "<u4").view("<f4")[0])
                    sites.append(_site(pc, w, lane, reg, 1 << bit))
                    out.append(O.SDC if sdc else O.MASKED)
                    within.append(sdc and _within(fv, float(gold[0])))
    assert any(within) and not all(x for x, o in zip(within, out) if o == O.SDC)
    _check(g, np.concatenate(sites), out, within)


def test_f64_pair_flips_against_numpy():
    """f64 (DADD into a register pair): a flip of low-word bit k moves the element
    by about 2^(k-52) relative, within 1e-6 for every k; a flip in the high word
    mostly by far more — the 8-byte element, not the 32-bit word, decides."""
    prog = P.vector_add_f64()
    g = O.Golden(prog)
    img = g.final_image()
    a, b = prog.view(img, "a", "<f8"), prog.view(img, "b", "<f8")
    sites, out, within = [], [], []
    for w, lane in ((0, 0), (3, 17), (15, 31)):
        t = w * 32 + lane
        gold = a[t:t + 1] + b[t:t + 1]
        for reg, shift in ((8, 0), (9, 32)):                       # DADD result: low / high word
            for bit in range(32):
                fu = int(gold.view("<u8")[0]) ^ (1 << (bit + shift))
                fv = float(np.array([fu], "<u8").view("<f8")[0])
                if np.isnan(fv):
                    fu = 0x7FFFFFFFFFFFFFFF
                sites.append(_site(15, w, lane, reg, 1 << bit))
                out.append(O.SDC)
                within.append(_within(fv, float(gold[0])))
        for reg, shift in ((8, 0), (9, 32)):                       # operand a (LDG.64)
            for bit in range(0, 32, 3):
                av = np.array([int(a[t:t + 1].view("<u8")[0]) ^ (1 << (bit + shift))], "<u8").view("<f8")
                with np.errstate(all="ignore"):
                    f = av + b[t:t + 1]
                fu = int(f.view("<u8")[0])
                if np.isnan(f[0]):
                    fu = 0x7FFFFFFFFFFFFFFF
                sdc = fu != int(gold.view("<u8")[0])
                sites.append(_site(11, w, lane, reg, 1 << bit))
                out.append(O.SDC if sdc else O.MASKED)
                within.append(sdc and _within(float(f[0]), float(gold[0])))
    assert any(within) and not all(within)
    _check(g, np.concatenate(sites), out, within)


@pytest.mark.parametrize("launch", [1, 2])
def test_chain_f32_propagated_against_numpy(launch):
    """Multi-launch (full mode): the corrupted word propagates through the later
    launches (y <- fma(y, 0.5, x)); the secondary class is decided on the final
    output y4 by the same definition."""
    n_inst, n = 4, 256
    prog = P.multi_instance_chain(n_inst=n_inst, n=n, block=64)
    g = O.Golden(prog)
    gold = g.final_image()
    x = prog.view(gold, "x", "<f4").astype(np.float64)
    y4g = prog.view(gold, f"y{n_inst}", "<f4")
    fp32 = O.G_FP32
    seen = set()
    for s in (launch * n + 5, launch * n + 77, launch * n + 200):
        site = g.locate(fp32, np.array([s], dtype=np.uint64))
        t = int(site["thread"][0])
        for bit in (0, 3, 9, 14, 20, 22, 25, 30, 31):
            site["mask"] = 1 << bit
            y = prog.view(gold, "y0", "<f4")
            for i in range(n_inst):
                with np.errstate(all="ignore"):
                    r = (y.astype(np.float64) * 0.5 + x).astype(np.float32)
                u = r.view("<u4").copy()
                u[np.isnan(r)] = 0x7FFFFFFF
                if i == launch:
                    u[t] ^= np.uint32(1 << bit)
                y = u.view("<f4")
            diff = np.flatnonzero(y.view("<u4") != y4g.view("<u4"))
            sdc = diff.size > 0
            win = sdc and all(_within(float(y[k]), float(y4g[k])) for k in diff)
            r = g.inject(site, O.MODE_FULL, rtol=RTOL)[0]
            assert r["outcome"] == (O.SDC if sdc else O.MASKED)
            assert bool(r["flags"] & O.SDC_WITHIN_TOL) == win, (s, bit)
            seen.add((sdc, win))
    assert (True, True) in seen and (True, False) in seen


def test_histogram_tol_counts_within_as_masked():
    sites = np.zeros(4, dtype=O.SITE_DTYPE)
    sites["group"], sites["bfm"] = GP, 0
    inj = np.zeros(4, dtype=O.INJ_DTYPE)
    inj["outcome"] = [O.SDC, O.SDC, O.MASKED, O.DUE]
    inj["flags"] = [O.SDC_WITHIN_TOL, 0, 0, 0]
    assert O.histogram(sites, inj)[GP, 0].tolist() == [1, 2, 1]
    assert O.histogram(sites, inj, tol=True)[GP, 0].tolist() == [2, 1, 1]
