"""GPU parity of the hybrid L+Z pattern routing vs. the oracle.

PAPER.md §III-E/F (Eqs. (8)-(14), the hybrid candidate set L1043-1092) and the
selection by two-pin HPWL (§IV-D); readings R23-R25.  Bar: batch ids,
seg (bend 0-3, ls, lt, straight), zmid (mid | lb << 16), per-net cost and the final
demand are bit-exact against oracle.route(..., hybrid=(t1, t2)).
"""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.helpers import design_from_json, load_golden

pytestmark = pytest.mark.gpu


def first_diff(a, b):
    idx = np.nonzero(a != b)[0]
    return None if len(idx) == 0 else (int(idx[0]), a[idx[0]], b[idx[0]], len(idx))


def check_hybrid(d, hybrid, r=None, demand0=None, min_z=1):
    import torch
    from paper_conf_date_liulzclly22_b200 import Router
    own = r is None
    if own:
        r = Router(d, device=0, hybrid=hybrid)
    r.reset_demand(None if demand0 is None else torch.from_numpy(demand0).cuda())
    nb = r.plan()
    r.route_all()
    b, nb, seg, cost, dem = r.results()
    zmid = r.zmids()
    o = Oracle(d)
    ob, onb = o.plan()
    assert nb == onb and np.array_equal(b, ob)
    oseg, ocost, odem, oz = o.route(ob, onb, demand=demand0, hybrid=hybrid, with_zmid=True)
    assert (oz >= 0).sum() >= min_z, "the case must exercise Z shapes"
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(zmid, oz), first_diff(zmid, oz)
    assert np.array_equal(cost, ocost), first_diff(cost, ocost)
    assert np.array_equal(dem, odem), first_diff(dem.ravel(), odem.ravel())
    if own:
        r.close()
    return int((oz >= 0).sum())


def test_w5_hand_worked_on_gpu():
    j = load_golden("W5.json")
    d = design_from_json(j)
    check_hybrid(d, tuple(j["hybrid"]))


@pytest.mark.parametrize("seed", range(10))
def test_random_small_hybrid(seed):
    L = [2, 3, 4, 5, 6, 9, 12, 16, 7, 9][seed]
    d = gen.random_small(seed=700 + seed, nx=40 + 5 * seed, ny=36 + 3 * seed, nlayers=L, num_nets=300, kmax=12,
                         literal_frac=0.3, caps=[1] + [2] * (L - 1))
    check_hybrid(d, (3 + seed % 3, 40 + 10 * seed))


def test_hybrid_big_nets_cta_path():
    """Nets > 32 nodes (CTA path: path walks, root-path transfer matrices) with hybrid edges."""
    d = gen.generate(nx=120, ny=110, nlayers=9, num_nets=300, seed=78, caps=gen.CAP9, pin_dist=1, kmin=30,
                     kmax=300, hpwl_base=30.0, hpwl_sigma=0.5, name="bignets_h")
    assert (d.net_sizes() > 32).sum() > 80
    check_hybrid(d, (4, 200), min_z=20)


def test_hybrid_nonuniform_directions():
    d = gen.random_small(seed=15, nx=50, ny=60, nlayers=7, num_nets=400, kmax=9)
    d.dir = np.array([1, 1, 0, 1, 0, 0, 1], np.uint8)
    rng = np.random.default_rng(3)
    d.via_cost = rng.integers(0, 90, size=6).astype(np.int32)
    d.ovf_weight = rng.integers(0, 9000, size=7).astype(np.int32)
    d.len_cost = 17
    d.logistic_slope = 0.37
    d.slack_clamp = 9
    check_hybrid(d, (3, 100))


@pytest.mark.parametrize("cfg,window", [("t1", (4, 200)), ("t5", (6, 300)), ("t5", (100, 500))])
def test_configs_hybrid(cfg, window):
    d = gen.make_config(cfg)
    check_hybrid(d, window, min_z=0 if window[0] >= 100 else 50)


def test_hybrid_route_batch_ex():
    import torch
    from paper_conf_date_liulzclly22_b200 import Router
    d = gen.make_config("t1")
    hyb = (4, 120)
    o = Oracle(d)
    ob, onb = o.plan()
    oseg, ocost, odem, oz = o.route(ob, onb, hybrid=hyb, with_zmid=True)
    r = Router(d, device=0, hybrid=hyb)
    r.reset_demand(None)
    r.seg.fill_(-1)
    r.cost.zero_()
    for b in range(onb):
        ids = torch.from_numpy(np.nonzero(ob == b)[0].astype(np.int32)).cuda()
        r.route_batch(ids)
    torch.cuda.synchronize()
    seg = r.seg.cpu().numpy().view(np.uint32)
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(r.zmids(), oz)
    assert np.array_equal(r.cost.cpu().numpy().view(np.uint32), ocost)
    assert np.array_equal(r.demand().cpu().numpy(), odem)
    r.close()


def test_hybrid_exchange_path_world1():
    from paper_conf_date_liulzclly22_b200 import Router
    from paper_conf_date_liulzclly22_b200 import fastgr as F
    d = gen.make_config("t5")
    r = Router(d, device=0, hybrid=(6, 300))
    F.fgr_comm_init(r.h, F.fgr_comm_unique_id(), 0, 1)
    check_hybrid(d, (6, 300), r=r, min_z=50)
    r.close()


def test_hybrid_window_toggle_and_l_only_unchanged():
    """Switching the window on one grid re-plans the tables; an empty window equals the L-only path."""
    from paper_conf_date_liulzclly22_b200 import Router
    from paper_conf_date_liulzclly22_b200 import fastgr as F
    d = gen.make_config("t1", num_nets=1500)
    r = Router(d, device=0, hybrid=(4, 80))
    check_hybrid(d, (4, 80), r=r)
    F.fgr_set_pattern(r.h, 10, 60)
    r.hybrid = (10, 60)
    check_hybrid(d, (10, 60), r=r)
    F.fgr_set_pattern(r.h, 1, 0)
    r.hybrid = (1, 0)
    n = check_hybrid(d, (1, 0), r=r, min_z=0)
    assert n == 0
    r.close()


def test_hybrid_t9_full_size():
    """BASELINE's headline config with the window that makes ~1% of the two-pin nets (tree edges)
    "medium", the share the paper reports for its t1 = 100, t2 = 500 (
    reading R23): t1 = 10, t2 = 500 selects 32k of t9's 3.04M edges."""
    d = gen.make_config("t9")
    check_hybrid(d, (10, 500), min_z=1000)
