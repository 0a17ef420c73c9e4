"""Pin the oracle's permanent / intermittent fault model.

PAPER.md:128-134 (Table III: a permanent fault is a fixed XOR mask on the
destination of every dynamic instance of one opcode executed in one lane of one
SM), :142-144 (the mask is applied to all destination registers), :254
(intermittent = a random subset of those instances).  Readings C-21 (CTA c runs
on SM c mod n_sm; a predicate destination flips iff bit 0 of the mask is set)
and C-22 (intermittent: the instance fires iff Philox(warp, step, rep) < q32).

Expected values come from numpy (IEEE f32 sums, the chain recurrence) and the
index arithmetic of the thread -> (CTA, lane) map, never from the oracle.
"""
import numpy as np
import pytest

import oracle as O
from fi_inputs import isa, programs as P


def pf(opcode, sm, lane, mask, n_sm, q32=0, seed=0):
    f = np.zeros(1, dtype=O.PFAULT_DTYPE)
    f[0] = (opcode, sm, lane, mask, q32, n_sm, seed)
    return f


@pytest.fixture(scope="module")
def c1():
    return O.Golden(P.vector_add(n=1000))


def _affected(n, block, sm, lane, n_sm):
    i = np.arange(n)
    return ((i // block) % n_sm == sm) & ((i % block) % 32 == lane)


@pytest.mark.parametrize("sm,lane,n_sm", [(1, 5, 3), (0, 0, 1), (3, 31, 4), (2, 7, 148)])
def test_permanent_fadd_xors_exactly_the_faulty_sm_lane(c1, sm, lane, n_sm):
    mask = 0x00400001
    k, img = c1.permanent_image(pf(isa.FADD, sm, lane, mask, n_sm))
    prog = c1.prog
    a, b, c = (prog.view(img, n, "<f4") for n in "abc")
    want = (a + b).view("<u4").copy()
    hit = _affected(1000, 256, sm, lane, n_sm)
    want[hit] ^= mask
    assert k == 0 and np.array_equal(c.view("<u4"), want)
    out = c1.inject_permanent(pf(isa.FADD, sm, lane, mask, n_sm))
    assert out["outcome"][0] == (O.SDC if hit.any() else O.MASKED)
    assert out["mask"][0] == mask


def test_permanent_on_idle_sm_or_absent_opcode_is_masked(c1):
    # grid 4: SM 7 of 148 runs no CTA; DMUL is not in the vector-add kernel
    for f in (pf(isa.FADD, 7, 0, 0xFFFFFFFF, 148), pf(isa.DMUL, 0, 0, 0xFFFFFFFF, 1),
              pf(isa.FADD, 0, 0, 0, 1)):
        k, img = c1.permanent_image(f)
        assert k == 0 and np.array_equal(img, c1.final_image())
        assert c1.inject_permanent(f)["outcome"][0] == O.MASKED


def test_permanent_isetp_flips_predicate_iff_mask_bit0(c1):
    # ISETP P0 = gid >= n guards the EXIT: a flipped P0 makes in-range threads exit
    # before their store (c stays 0) and lets the 24 out-of-range lanes run on:
    # thread 1000+j (lane 8+j of warp 31) then loads a[1000+j], past the buffer
    k, img = c1.permanent_image(pf(isa.ISETP, 3, 9, 1, 4))
    assert k == 2                                  # unmapped load (C-9)
    assert c1.inject_permanent(pf(isa.ISETP, 3, 9, 1, 4))["outcome"][0] == O.DUE
    # lane 3 of SM 3: thread 768 + 32w + 3 < 1000 only; no out-of-range lane hit
    k, img = c1.permanent_image(pf(isa.ISETP, 3, 3, 1, 4))
    hit = _affected(1000, 256, 3, 3, 4)
    want = (c1.prog.view(img, "a", "<f4") + c1.prog.view(img, "b", "<f4")).view("<u4").copy()
    want[hit] = 0
    assert k == 0 and np.array_equal(c1.prog.view(img, "c", "<u4"), want)
    # mask without bit 0 leaves predicates alone
    k, img = c1.permanent_image(pf(isa.ISETP, 3, 3, 0xFFFFFFFE, 4))
    assert k == 0 and np.array_equal(img, c1.final_image())
    assert hit.sum() == 8                          # 768 + 32w + 3 < 1000 for w = 0..7


def test_permanent_address_fault_is_due_and_potential_due_unchecked(c1):
    # IMAD_WIDE writes the a-pointer pair: XOR 2 into both words -> misaligned
    # (and unmapped) load: DUE; with unchecked error semantics (row f4) the
    # faulting warps stop and the rest of c stands
    f = pf(isa.IMAD_WIDE, 0, 4, 2, 4)
    r = c1.inject_permanent(f)
    assert r["outcome"][0] == O.DUE and r["fault_kind"][0] in (1, 2)
    r = c1.inject_permanent(f, mode=O.UNCHECKED)
    assert r["outcome"][0] == O.SDC and r["flags"][0] & O.POTENTIAL_DUE
    k, img = c1.permanent_image(f, mode=O.UNCHECKED)
    cv = c1.prog.view(img, "c", "<u4")
    gold = c1.prog.view(c1.final_image(), "c", "<u4")
    # warps of CTA 0 stop at the faulting load, before any store (C-14 keeps
    # stores of a warp that faulted earlier; here there are none)
    assert (cv[:256] == 0).all() and np.array_equal(cv[256:], gold[256:])


def test_permanent_fault_persists_across_instances():
    # chain: y_{i+1} = fma(y_i, 0.5, x); every launch of FFMA on the faulty SM
    # lane re-applies the mask (numpy recurrence)
    n, blk, n_inst = 256, 64, 4
    g = O.Golden(P.multi_instance_chain(n_inst=n_inst, n=n, block=blk))
    mask, sm, lane, nsm = 0x80000000, 2, 17, 3
    k, img = g.permanent_image(pf(isa.FFMA, sm, lane, mask, nsm))
    x = g.prog.view(img, "x", "<f4").astype(np.float64)
    y = g.prog.view(img, "y0", "<f4")
    hit = _affected(n, blk, sm, lane, nsm)
    for i in range(n_inst):
        y = (y.astype(np.float64) * 0.5 + x).astype(np.float32)
        u = y.view("<u4").copy()
        u[hit] ^= mask
        y = u.view("<f4")
        assert np.array_equal(g.prog.view(img, f"y{i + 1}", "<u4"), u)
    assert k == 0 and hit.sum() == 2                # CTA 2 of 4, two warps of 64 threads
    assert g.inject_permanent(pf(isa.FFMA, sm, lane, mask, nsm))["outcome"][0] == O.SDC


def test_intermittent_fires_on_a_q_fraction_and_is_replica_seeded():
    n, blk = 32768, 256
    g = O.Golden(P.vector_add(n=n, grid=n // blk, block=blk))
    gold = g.prog.view(g.final_image(), "c", "<u4")
    lane, mask = 6, 0x10

    def fired(q32, rep, seed=5):
        k, img = g.permanent_image(pf(isa.FADD, 0, lane, mask, 1, q32=q32, seed=seed), rep=rep)
        d = g.prog.view(img, "c", "<u4") ^ gold
        assert k == 0 and set(np.unique(d)) <= {0, mask}
        hit = d != 0
        assert not (hit & ~_affected(n, blk, 0, lane, 1)).any()
        return hit

    m = _affected(n, blk, 0, lane, 1).sum()          # 1024 candidate instances
    h0, h1 = fired(1 << 31, 0), fired(1 << 31, 1)
    for h in (h0, h1):                               # Binomial(1024, 1/2): 6 sigma = 96
        assert abs(int(h.sum()) - m // 2) < 96
    assert not np.array_equal(h0, h1)                # replicas draw independently
    assert np.array_equal(h0, fired(1 << 31, 0))     # and deterministically
    assert abs(int(fired(1 << 30, 0).sum()) - m // 4) < 84
    assert fired(1, 0).sum() == 0                    # P = 2^-32 per instance
    assert fired(0xFFFFFFFF, 3).sum() == m           # P = 1 - 2^-32
