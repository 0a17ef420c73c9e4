"""Parity at BASELINE.json's full size (C2: SGEMM 4096^3, 10,000 replicas) in
the launch configuration bench.py times (campaign.Campaign.step).

The oracle cannot re-run all 8,192 warps in a test, so it checks:
  * counts and record totals against the hand-derived closed form;
  * every one of the 10,000 draws (s, u_dst, u_bit) against its own Philox+Lemire;
  * every site's warp against the closed-form per-warp count, and its mask;
  * a stratified sample of replicas fully: the oracle selects the site itself
    (draw -> warp -> enumeration inside the warp) and injects it warp-locally;
    site fields, before/after/mask, fault kind and outcome must be identical.
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
