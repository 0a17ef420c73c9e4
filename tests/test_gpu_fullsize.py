"""Parity at BASELINE.json's full size (C2: SGEMM 4096^3, 10,000 replicas) in
the launch configuration bench.py times (campaign.Campaign.step).

Checks:
  * counts and record totals against the hand-derived closed form;
  * every one of the 10,000 draws (s, u_dst, u_bit) against its own Philox+Lemire;
  * every site's warp against the closed-form per-warp count, and its mask;
  * ALL 10,000 replicas against the oracle: its own golden run of the whole
    C2 program (orc_golden_run without a kept trace: per-warp counts and the
    golden final image, PAPER.md:72 step (1)), its own selection (the warp from
    the per-warp counts, the rank inside it by re-interpreting that warp, C-3)
    and warp-local injection classified against that golden image
    (C-14) — every site field, before/after/mask, fault kind/pc
    and outcome identical, no replica left undecided;
  * the GPU golden final image equals the oracle's byte for byte;
  * the golden run's own (fused) profile equals K1's scan of its trace;
  * a stratified sample again through build_site / inject_local (the checker
    without a golden handle, pinned in tests/test_oracle_pins_local.py).
"""
import numpy as np
import pytest

import oracle as O
from closed_forms import sgemm_closed_form, sgemm_per_thread, GP
from fi_inputs import programs as P

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def camp():
    from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign
    c = Campaign(P.c2(full=True), P.CAMPAIGN_SEED[2], [GP], [0, 1, 2, 3], 10000)
    c.step()
    c.check()
    return c


@pytest.fixture(scope="module")
def oracle_c2(camp):
    return O.Golden(camp.prog, keep_trace=False)


def test_c2_oracle_golden_run(camp, oracle_c2):
    want, nrec = sgemm_closed_form(4096, 4096, 4096)
    assert oracle_c2.counts()[0].tolist() == want and oracle_c2.n_records == nrec
    assert np.array_equal(camp.gt.image.cpu().numpy(), oracle_c2.final_image())
    assert np.array_equal(camp.gt.warp_len.cpu().numpy().astype(np.uint64), oracle_c2.warp_len())


def test_c2_all_10000_replicas_vs_oracle(camp, oracle_c2):
    """Every replica of the headline campaign, element by element (no sample,
    no undecided escape): sites, injected values, faults and outcomes."""
    sites = camp.sites_np()
    inj = camp.inj_np()
    osites = oracle_c2.select(P.CAMPAIGN_SEED[2], [GP], [0, 1, 2, 3], 0, 10000)
    for n in osites.dtype.names:
        assert (osites[n] == sites[n]).all(), n
    oi = oracle_c2.inject(osites, O.MODE_WARP_LOCAL)
    for f in ("before", "after", "mask", "fault_kind", "outcome", "flags"):
        bad = np.flatnonzero(oi[f] != inj[f])
        assert bad.size == 0, (f, bad[:10].tolist())
    fk = oi["fault_kind"] > 0
    assert (oi["fault_pc"][fk] == inj["fault_pc"][fk]).all()
    assert (inj["overflow"] == 0).all()
    h = camp.hist.cpu().numpy()
    assert (h == O.histogram(osites, oi).astype(np.int64)).all()
    assert set(np.unique(oi["outcome"]).tolist()) == {0, 1, 2}


def test_c2_golden_run_profile(camp):
    """The profile counted inside the JIT golden pass 2 (record templates, chunk
    crossings inside a block, step mode) equals K1's scan of the written trace."""
    from paper_conf_dsn_0002hsvk21_b200 import fi
    gi, gc = fi.golden_profile(camp.gt)
    assert np.array_equal(gi.cpu().numpy(), camp.inst_counts.cpu().numpy())
    assert np.array_equal(gc.cpu().numpy(), camp.chunk_counts.cpu().numpy())


def test_c2_counts_closed_form(camp):
    want, nrec = sgemm_closed_form(4096, 4096, 4096)
    assert camp.inst_counts.cpu().numpy()[0].tolist() == want
    assert camp.gt.n_rec == nrec


def test_c2_all_draws_and_sites(camp):
    sites = camp.sites_np()
    N = sgemm_closed_form(4096, 4096, 4096)[0][GP]
    per_warp = 32 * sgemm_per_thread(4096)[GP]
    seed = P.CAMPAIGN_SEED[2]
    for j in range(len(sites)):
        s, ud, ub, _ = O.draw(seed, j, N)
        assert (int(sites["s"][j]), int(sites["u_dst"][j]), int(sites["u_bit"][j])) == (s, ud, ub), j
        assert int(sites["warp"][j]) == s // per_warp
        assert int(sites["mask"][j]) == O.mask(j % 4, ub)
    assert (sites["bfm"] == np.arange(len(sites)) % 4).all()


def test_c2_sampled_replicas(camp):
    prog = camp.prog
    sites = camp.sites_np()
    inj = camp.inj_np()
    N = sgemm_closed_form(4096, 4096, 4096)[0][GP]
    per_warp = 32 * sgemm_per_thread(4096)[GP]
    rng = np.random.Generator(np.random.PCG64(7))
    js = sorted(set(rng.choice(10000, 44, replace=False).tolist()) | {0, 1, 2, 3})
    # make sure DUE and (if any) Masked replicas are represented
    for o in (0, 2):
        js += np.flatnonzero(inj["outcome"] == o)[:6].tolist()
    js = sorted(set(js))
    orows = np.concatenate([O.build_site(prog, P.CAMPAIGN_SEED[2], j, GP, j % 4, per_warp, N) for j in js])
    names = [n for n in orows.dtype.names if n != "pad"]
    for n in names:
        assert (orows[n] == sites[n][js]).all(), n
    oi, decided = O.inject_local(prog, orows)
    gi = inj[js]
    for f in ("before", "after", "mask", "fault_kind"):
        assert (oi[f] == gi[f]).all(), f
    assert (oi["fault_pc"][oi["fault_kind"] > 0] == gi["fault_pc"][gi["fault_kind"] > 0]).all()
    assert decided.mean() > 0.8
    assert (oi["outcome"][decided] == gi["outcome"][decided]).all()


def test_c2_histogram_accounts(camp):
    h = camp.hist.cpu().numpy()
    inj = camp.inj_np()
    assert int(h.sum()) == 10000
    for o in range(3):
        assert int(h[..., o].sum()) == int((inj["outcome"] == o).sum())
    assert not inj["overflow"].any()
