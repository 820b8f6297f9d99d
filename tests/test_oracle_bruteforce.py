"""Oracle DP vs. brute-force enumeration of every per-edge (bend, ls, lt) assignment.

Pins Eqs. (1)-(4) and the span-enumeration reading R3 of
Eq. (2): on tiny trees the DP minimum must equal the minimum over all 3-D
L-shape routings (2*|H|*|V| options per bent edge, |dir| per straight edge)
with via stacks over the hull of every node's incident layers, and the DP's
chosen route must re-cost to its reported value.
"""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.helpers import PyCost, brute_force_min, route_cost


def _tiny_designs():
    out = []
    for seed in range(40):
        L = 2 + seed % 4          # 2..5 layers
        d = gen.random_small(seed=1000 + seed, nx=7, ny=6, nlayers=L, num_nets=6, kmax=4,
                             literal_frac=0.4, caps=[1] * L)
        out.append(d)
    return out


@pytest.mark.parametrize("d", _tiny_designs(), ids=lambda d: d.name)
def test_dp_equals_bruteforce(d):
    o = Oracle(d)
    rng = np.random.default_rng(d.seed)
    # random congestion so the logistic term matters (slack around 0)
    demand = rng.integers(0, 3, size=(d.nlayers, d.ny, d.nx)).astype(np.int32)
    pc = PyCost(d, demand)
    checked = 0
    for n in range(d.num_nets):
        m = d.node_offset[n + 1] - d.node_offset[n]
        if m < 2 or m > 5:
            continue
        seg, cost = o.route_net(n, demand)
        bf = brute_force_min(d, n, demand)
        assert cost == bf, (d.name, n)
        a = d.node_offset[n]
        assert route_cost(d, pc, n, [None] + list(seg[a + 1:a + m])) == cost
        assert o.recost_net(n, demand, seg) == cost
        checked += 1
    assert checked > 0


def test_bruteforce_with_pin_spans_and_vias():
    """Multi-layer pin spans and unequal via costs (hull reading R3/R4)."""
    for seed in range(30):
        d = gen.random_small(seed=5000 + seed, nx=6, ny=6, nlayers=5, num_nets=4, kmax=4, literal_frac=0.0)
        rng = np.random.default_rng(seed)
        d.via_cost = rng.integers(0, 50, size=4).astype(np.int32)
        d.ovf_weight = rng.integers(0, 5000, size=5).astype(np.int32)
        d.len_cost = int(rng.integers(1, 100))
        lo = rng.integers(0, 5, size=d.num_nodes)
        hi = np.minimum(4, lo + rng.integers(0, 3, size=d.num_nodes))
        steiner = rng.random(d.num_nodes) < 0.3
        d.pin_lo = np.where(steiner, -1, lo).astype(np.int8)
        d.pin_hi = np.where(steiner, -1, hi).astype(np.int8)
        o = Oracle(d)
        demand = rng.integers(0, 4, size=(5, d.ny, d.nx)).astype(np.int32)
        for n in range(d.num_nets):
            m = d.node_offset[n + 1] - d.node_offset[n]
            if m < 2 or m > 5:
                continue
            _, cost = o.route_net(n, demand)
            assert cost == brute_force_min(d, n, demand), (seed, n)


def test_straight_edge_reading_R7():
    """Reading R7: a straight tree edge takes the single candidate ls = lt with
    one leg.  Pinned against the general degenerate L shapes (a zero-length leg on any layer at an
    endpoint plus the bend via, on both bends): over random tiny trees with pins, Steiner nodes,
    unequal via costs and congestion, the minimum over the general candidate set equals the
    oracle's cost (sub-additivity of the via stack makes the extra candidates never better)."""
    checked = straight = 0
    for seed in range(60):
        L = 3 + seed % 3
        d = gen.random_small(seed=7000 + seed, nx=6, ny=5, nlayers=L, num_nets=5, kmax=4, literal_frac=0.3,
                             caps=[1] * L)
        rng = np.random.default_rng(seed)
        d.via_cost = rng.integers(0, 60, size=L - 1).astype(np.int32)
        o = Oracle(d)
        demand = rng.integers(0, 3, size=(L, d.ny, d.nx)).astype(np.int32)
        for n in range(d.num_nets):
            a, m = d.node_offset[n], d.node_offset[n + 1] - d.node_offset[n]
            if m < 2 or m > 4:
                continue
            ns = sum(1 for i in range(1, m) if d.x[a + i] == d.x[a + d.parent[a + i]] or
                     d.y[a + i] == d.y[a + d.parent[a + i]])
            _, cost = o.route_net(n, demand)
            assert cost == brute_force_min(d, n, demand, general_straight=True), (seed, n)
            checked += 1
            straight += ns
    assert checked > 40 and straight > 20, (checked, straight)
