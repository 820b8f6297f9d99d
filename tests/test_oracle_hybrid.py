"""Oracle pins for the hybrid L+Z pattern routing.

PAPER.md §III-E/F: Z-shape cost Eq. (8) (L831-842), candidate flows Eqs. (9),
(11)-(14) (L848-1032), merge Eq. (10) (L864-872), the hybrid candidate set (the
two L shapes + the Z shapes, L1043-1092) and the selection by two-pin HPWL
(§IV-D).  Readings R23-R25.  Pins:
  * W5 (tests/golden/W5.json): hand-worked values of a Z that beats both L's;
  * brute force over every per-edge route (L and Z) with node via hulls;
  * closed form W4 with Z shapes (monotone paths: total = LEN * Manhattan length);
  * invariants: empty window == L only; hybrid cost <= L-only cost on the same
    demand; chosen route re-costs to the reported value; demand = recount.
"""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.helpers import (PyCost, brute_force_min, design_from_json, load_golden, recount_demand, route_cost,
                           seg_fields)


def test_w5_hand_worked():
    j = load_golden("W5.json")
    d = design_from_json(j)
    o = Oracle(d)
    b, nb = o.plan()
    seg, cost, dem, zmid = o.route(b, nb, hybrid=tuple(j["hybrid"]), with_zmid=True)
    assert list(cost) == j["expect"]["total"]
    assert seg[0] == 0xFFFFFFFF
    assert seg_fields(seg[1]) == j["expect"]["seg"][0][1]
    assert list(zmid) == j["expect"]["zmid"][0]
    want = np.zeros_like(dem)
    for l, y, x in j["expect"]["demand_plus_one"]:
        want[l, y, x] += 1
    assert np.array_equal(dem, want)
    # L only: the paper's FastGRL candidate set
    seg_l, cost_l, _ = o.route(b, nb)
    assert list(cost_l) == j["expect"]["l_only_total"]
    assert seg_fields(seg_l[1]) == j["expect"]["l_only_seg"][0][1]
    # the edge's HPWL (5) outside the window -> L only
    seg_o, cost_o, _, z_o = o.route(b, nb, hybrid=(6, 10), with_zmid=True)
    assert list(cost_o) == j["expect"]["l_only_total"] and list(z_o) == [-1, -1]
    # independent re-costing of the chosen Z route
    pc = PyCost(d, np.zeros_like(dem))
    assert route_cost(d, pc, 0, [None, seg[1]], [None, int(zmid[1])]) == 384
    assert o.recost_net(0, np.zeros_like(dem), seg, zmid) == 384


def _tiny(seed, L):
    return gen.random_small(seed=seed, nx=6, ny=6, nlayers=L, num_nets=8, kmax=3, literal_frac=0.4,
                            caps=[1] * L)


@pytest.mark.parametrize("seed", range(24))
def test_hybrid_dp_equals_bruteforce(seed):
    """The DP over hybrid edges = the minimum over every per-edge L/Z route (Eq. (10) merged into Eq. (2))."""
    L = 2 + seed % 3
    d = _tiny(3000 + seed, L)
    rng = np.random.default_rng(seed)
    if seed % 2:
        d.via_cost = rng.integers(0, 50, size=L - 1).astype(np.int32)
        d.len_cost = int(rng.integers(1, 100))
    o = Oracle(d)
    demand = rng.integers(0, 3, size=(L, d.ny, d.nx)).astype(np.int32)
    pc = PyCost(d, demand)
    hyb = (2, 12)
    checked = 0
    for n in range(d.num_nets):
        a, m = d.node_offset[n], d.node_offset[n + 1] - d.node_offset[n]
        if m < 2 or m > 3:
            continue
        zmid = np.full(d.num_nodes, -1, np.int32)
        seg, cost = o.route_net(n, demand, hybrid=hyb, zmid=zmid)
        assert cost == brute_force_min(d, n, demand, hybrid=hyb), (seed, n)
        assert route_cost(d, pc, n, [None] + list(seg[a + 1:a + m]), [None] + list(zmid[a + 1:a + m])) == cost
        assert o.recost_net(n, demand, seg, zmid) == cost
        _, cost_l = o.route_net(n, demand)
        assert cost <= cost_l
        checked += 1
    assert checked > 0


def test_hybrid_closed_form_w4():
    """VIA = 0, W = 0: every L and Z route is monotone, so total = LEN * sum of Manhattan lengths (W4)."""
    d = gen.random_small(seed=77, nx=30, ny=30, nlayers=5, num_nets=60, kmax=5, literal_frac=0.3)
    d.via_cost = np.zeros(4, np.int32)
    d.ovf_weight = np.zeros(5, np.int32)
    o = Oracle(d)
    b, nb = o.plan()
    seg, cost, dem, zmid = o.route(b, nb, hybrid=(2, 60), with_zmid=True)
    for n in range(d.num_nets):
        a, e = d.node_offset[n], d.node_offset[n + 1]
        wl = 0
        for v in range(a + 1, e):
            u = a + d.parent[v]
            wl += abs(int(d.x[v]) - int(d.x[u])) + abs(int(d.y[v]) - int(d.y[u]))
        assert int(cost[n]) == d.len_cost * wl
    assert np.array_equal(dem, recount_demand(d, seg, zmid=zmid))


def test_hybrid_stage_invariants():
    """Whole stage with Z shapes: some Z chosen, demand = recount, costs re-cost on the demand at their
    batch's start, sequential-within-batch == batch-synchronous, an empty window == L only."""
    d = gen.random_small(seed=4242, nx=40, ny=32, nlayers=5, num_nets=220, kmax=6, literal_frac=0.3,
                         caps=[1, 1, 1, 1, 1])
    o = Oracle(d)
    b, nb = o.plan()
    hyb = (3, 40)
    seg, cost, dem, hashes, zmid = o.route(b, nb, hybrid=hyb, hashes=True, with_zmid=True)
    assert (zmid >= 0).sum() > 5
    bends = np.array([seg_fields(s)["bend"] for s in seg if s != 0xFFFFFFFF])
    assert (bends >= 2).sum() == (zmid >= 0).sum()
    assert np.array_equal(dem, recount_demand(d, seg, zmid=zmid))
    seg2, cost2, dem2, h2, z2 = o.route(b, nb, hybrid=hyb, sequential=True, hashes=True, with_zmid=True)
    assert np.array_equal(seg, seg2) and np.array_equal(cost, cost2) and np.array_equal(zmid, z2)
    assert np.array_equal(hashes, h2)
    # per-batch re-costing on the demand at the start of each batch
    cur = o.zero_demand()
    for bb in range(nb):
        nets = np.nonzero(b == bb)[0]
        for n in nets:
            assert o.recost_net(int(n), cur, seg, zmid) == int(cost[n])
        for n in nets:
            o.commit_net(int(n), seg, cur, zmid)
    assert np.array_equal(cur, dem)
    # empty window (t1 > t2) and a window no edge reaches: identical to L only
    seg_l, cost_l, dem_l = o.route(b, nb)
    for win in [(5, 4), (10_000, 20_000)]:
        s3, c3, d3, z3 = o.route(b, nb, hybrid=win, with_zmid=True)
        assert np.array_equal(s3, seg_l) and np.array_equal(c3, cost_l) and np.array_equal(d3, dem_l)
        assert (z3 == -1).all()
