"""Oracle invariants that hold at any size (SURVEY.md §8(c) 'What pins each part')."""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.helpers import (boxes_touch, net_bbox, recount_demand, sort_order, PyCost, route_cost)


def _designs():
    ds = [gen.make_config("tiny"), gen.make_config("t1", num_nets=600)]
    ds += [gen.random_small(seed=s, nx=16, ny=12, nlayers=3 + s % 3, num_nets=60, kmax=6) for s in range(4)]
    return ds


@pytest.fixture(scope="module", params=_designs(), ids=lambda d: d.name)
def routed(request):
    d = request.param
    o = Oracle(d)
    b, nb = o.plan()
    seg, cost, dem, hashes = o.route(b, nb, hashes=True)
    return d, o, b, nb, seg, cost, dem


def test_batches_conflict_free_and_first_fit(routed):
    """Alg. 1: no two nets of one batch conflict (L504), and a
    net lands in batch b only if every earlier batch already holds a conflicting
    net that precedes it in the sorted order (first fit, SURVEY.md §8(c) proof)."""
    d, o, b, nb, *_ = routed
    order = sort_order(d)
    boxes = {n: net_bbox(d, n) for n in order}
    rank = {n: r for r, n in enumerate(order)}
    for n in range(d.num_nets):
        if d.node_offset[n + 1] - d.node_offset[n] < 2:
            assert b[n] == -1
    used = set(b[b >= 0])
    assert used == set(range(nb))
    for i in order:
        seen = set()
        for j in order[:rank[i]]:
            if boxes_touch(boxes[i], boxes[j]):
                assert b[j] != b[i], (i, j)
                seen.add(int(b[j]))
        # batch(i) = mex of the batches of earlier conflicting nets
        mex = 0
        while mex in seen:
            mex += 1
        assert b[i] == mex


def test_demand_equals_committed_legs(routed):
    d, o, b, nb, seg, cost, dem = routed
    assert np.array_equal(recount_demand(d, seg), dem)


def test_sequential_equals_batch_synchronous(routed):
    """Nets of one batch are independent (bbox-disjoint, reading R13)."""
    d, o, b, nb, seg, cost, dem = routed
    seg2, cost2, dem2 = o.route(b, nb, sequential=True)
    assert np.array_equal(seg, seg2) and np.array_equal(cost, cost2) and np.array_equal(dem, dem2)


def test_cost_is_recost_at_batch_start(routed):
    """Per-net reported cost = independent re-costing of its route on the demand
    at the start of its batch (batches run in sequence)."""
    d, o, b, nb, seg, cost, dem = routed
    demand = o.zero_demand()
    for bb in range(nb):
        nets = np.nonzero(b == bb)[0]
        pc = PyCost(d, demand) if bb < 3 else None
        for n in nets:
            assert o.recost_net(n, demand, seg) == cost[n]
            if pc is not None:
                a, e = d.node_offset[n], d.node_offset[n + 1]
                assert route_cost(d, pc, n, [None] + list(seg[a + 1:e])) == cost[n]
        for n in nets:
            o.commit_net(n, seg, demand)
    assert np.array_equal(demand, dem)


def test_closed_form_no_via_no_congestion():
    """W4: VIA=0, W=0 -> Total = LEN * sum of Manhattan edge lengths."""
    for s in range(3):
        d = gen.random_small(seed=300 + s, nx=20, ny=20, nlayers=5, num_nets=80, kmax=8)
        d.via_cost = np.zeros(4, np.int32)
        d.ovf_weight = np.zeros(5, np.int32)
        o = Oracle(d)
        b, nb = o.plan()
        _, cost, _ = o.route(b, nb)
        for n in range(d.num_nets):
            a, e = d.node_offset[n], d.node_offset[n + 1]
            wl = sum(abs(int(d.x[v]) - int(d.x[a + d.parent[v]])) + abs(int(d.y[v]) - int(d.y[a + d.parent[v]]))
                     for v in range(a + 1, e))
            assert cost[n] == 64 * wl


def _reroot(d, n, new_root):
    """Return node arrays of net n re-rooted at local node new_root, in DFS preorder."""
    a, e = d.node_offset[n], d.node_offset[n + 1]
    m = e - a
    adj = [[] for _ in range(m)]
    for i in range(1, m):
        p = int(d.parent[a + i])
        adj[i].append(p); adj[p].append(i)
    order, par, stack, seen = [], {}, [(new_root, -1)], set()
    while stack:
        v, p = stack.pop()
        if v in seen:
            continue
        seen.add(v); order.append(v); par[v] = p
        for w in sorted(adj[v], reverse=True):
            if w not in seen:
                stack.append((w, v))
    idx = {v: k for k, v in enumerate(order)}
    return ([int(d.x[a + v]) for v in order], [int(d.y[a + v]) for v in order],
            [int(d.pin_lo[a + v]) for v in order], [int(d.pin_hi[a + v]) for v in order],
            [-1 if par[v] < 0 else idx[par[v]] for v in order])


def test_reroot_invariance():
    """Reading R20: the optimal cost does not depend on the chosen root (same set of
    physical L-routes and node hulls)."""
    rng = np.random.default_rng(7)
    for s in range(6):
        d = gen.random_small(seed=700 + s, nx=12, ny=12, nlayers=4, num_nets=15, kmax=6)
        o = Oracle(d)
        demand = rng.integers(0, 3, size=(4, 12, 12)).astype(np.int32)
        for n in range(d.num_nets):
            m = d.node_offset[n + 1] - d.node_offset[n]
            if m < 3:
                continue
            _, c0 = o.route_net(n, demand)
            for r in range(1, m):
                x, y, lo, hi, par = _reroot(d, n, r)
                d2 = d.subset([n])
                d2.x, d2.y = np.array(x, np.int16), np.array(y, np.int16)
                d2.pin_lo, d2.pin_hi = np.array(lo, np.int8), np.array(hi, np.int8)
                d2.parent = np.array(par, np.int32)
                _, c1 = Oracle(d2).route_net(0, demand)
                assert c1 == c0, (s, n, r)


def test_validation_rejects_bad_trees():
    d = gen.random_small(seed=1, num_nets=5)
    o = Oracle(d)
    assert o.validate()[0] == 0
    bad = d.subset(range(5))
    a = bad.node_offset[2]
    if bad.node_offset[3] - a >= 2:
        bad.parent[a + 1] = 1      # self/forward parent
        assert Oracle(bad).validate() == (1, 2)
    bad2 = d.subset(range(5))
    bad2.x[0] = bad2.nx            # out of grid
    assert Oracle(bad2).validate() == (1, 0)
