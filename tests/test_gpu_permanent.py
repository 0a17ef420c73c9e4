"""GPU parity of permanent / intermittent fault injection.

fi_inject_permanent (K7 in permanent mode: every warp of every CTA on the faulty
SM re-executed against the overlay, in every instance that runs the opcode)
against the oracle's whole-program re-run with the fault armed (the definition,
PAPER.md:128-134, :142-144, :254; readings C-21, C-22).  Outcome, flags, mask
and fault kind must be identical; the opcode-weighted histogram
must equal the oracle outcomes weighted by the same table.
"""
import numpy as np
import pytest
import torch

import oracle as O
from fi_inputs import isa, programs as P

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    from paper_conf_dsn_0002hsvk21_b200 import fi
    return fi


def _faults(prog, n, seed, intermittent):
    rng = np.random.default_rng(seed)
    present = np.unique(prog.code["op"]).astype(np.uint32)
    f = np.zeros(n, dtype=O.PFAULT_DTYPE)
    ops = rng.choice(present, n)
    other = rng.random(n) < 0.1                      # any opcode, possibly absent from the program
    ops[other] = rng.integers(0, isa.N_OPCODES, other.sum())
    f["opcode"] = ops
    f["n_sm"] = rng.choice(np.array([0, 1, 2, 3, 4, 7, 148], dtype=np.uint32), n)
    nsm = np.where(f["n_sm"] == 0, 148, f["n_sm"])
    f["sm"] = rng.integers(0, 1 << 30, n) % np.minimum(nsm, 8)
    f["lane"] = rng.integers(0, 32, n)
    kind = rng.integers(0, 4, n)
    one = np.uint32(1) << rng.integers(0, 32, n).astype(np.uint32)
    two = one | (np.uint32(1) << rng.integers(0, 32, n).astype(np.uint32))
    f["mask"] = np.select([kind == 0, kind == 1, kind == 2], [one, two, rng.integers(0, 1 << 32, n, dtype=np.uint64)
                                                              .astype(np.uint32)], np.uint32(1))
    if intermittent:
        f["q32"] = rng.integers(1, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
        f["seed"] = rng.integers(0, 1 << 63, n, dtype=np.uint64)
    return f


def _parity(F, prog, n, seed, intermittent=False, unchecked=False, batched=False):
    g = O.Golden(prog)
    dp = F.DeviceProgram(prog)
    gt = F.golden_run(dp)
    f = _faults(prog, n, seed, intermittent)
    opw = np.arange(1, F.FI_NOPS + 1, dtype=np.int64) * 3
    inj = F.inject_permanent_batched if batched else F.inject_permanent
    out, hist = inj(gt, f, op_weights=torch.from_numpy(opw).cuda(), unchecked=unchecked)
    gi = F.as_numpy(out, F.INJ_DTYPE, n)
    oi = g.inject_permanent(f, mode=O.MODE_FULL | (O.UNCHECKED if unchecked else 0))
    bad = np.nonzero(gi["outcome"] != oi["outcome"])[0]
    assert len(bad) == 0, (bad[:8], f[bad[:8]], gi["outcome"][bad[:8]], oi["outcome"][bad[:8]])
    for k in ("flags", "mask", "fault_kind", "fault_pc"):
        assert (gi[k] == oi[k]).all(), k
    want = np.zeros(3, dtype=np.int64)
    np.add.at(want, oi["outcome"].astype(np.int64), opw[f["opcode"] % F.FI_NOPS])
    assert np.array_equal(hist.cpu().numpy(), want)
    return oi


@pytest.mark.parametrize("maker", [lambda: P.vector_add(n=1000),
                                   lambda: P.multi_instance_chain(5),
                                   lambda: P.multi_instance_chain(4, n=300, block=96),
                                   lambda: P.fuzz_program(7, n_ops=90)])
def test_permanent_parity(F, maker):
    oi = _parity(F, maker(), 160, 11)
    assert len(np.unique(oi["outcome"])) >= 2


def test_permanent_parity_unchecked(F):
    _parity(F, P.vector_add(n=1000), 160, 12, unchecked=True)
    _parity(F, P.multi_instance_chain(4, n=300, block=96), 120, 13, unchecked=True)


def test_intermittent_parity(F):
    _parity(F, P.vector_add(n=1000), 160, 14, intermittent=True)
    _parity(F, P.multi_instance_chain(5), 120, 15, intermittent=True)


def test_permanent_parity_sgemm_mini(F):
    _parity(F, P.c2(full=False), 48, 16)


def test_permanent_parity_c3_mini(F):
    oi = _parity(F, P.c3(full=False), 64, 17)
    assert (oi["outcome"] == O.SDC).any()


@pytest.mark.parametrize("maker,intermittent,unchecked", [
    (lambda: P.vector_add(n=1000), False, False),
    (lambda: P.multi_instance_chain(5), False, False),
    (lambda: P.multi_instance_chain(4, n=300, block=96), True, True),
    (lambda: P.scatter_chain(), False, False),
    (lambda: P.c3(full=False), False, False),
])
def test_permanent_parity_k8(F, maker, intermittent, unchecked):
    """Rows f2/f3 on K8 (fi_inject_permanent_batched) against the oracle."""
    _parity(F, maker(), 120, 21, intermittent=intermittent, unchecked=unchecked, batched=True)


def test_permanent_parity_k8_c4_mini(F):
    from fi_inputs import resnet as R
    oi = _parity(F, R.c4(full=False), 64, 22, batched=True)
    assert (oi["outcome"] == O.SDC).any()
