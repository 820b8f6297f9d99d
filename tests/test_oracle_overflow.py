"""Oracle pins for the rip-up extraction and the ordered task graph.

PAPER.md §III-A L398-402 and §III-G L1109-1115 (the nets with violations are
ripped up), §III-B L414-466 (task conflict graph, root task batch by one pass of
Algorithm 1, root -> non-root, else smaller task ID first).  Readings R26-R27.
Pins: hand-worked OV1 / TG1 (tests/golden/), an independent Python recount of
the overflowed edges and violating nets, and for the task graph a pairwise brute
force plus the first-fit characterisation of the root batch (colour 0).
"""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.helpers import (boxes_touch, design_from_json, legs_of_edge, load_golden, net_bbox)


def test_ov1_hand_worked():
    j = load_golden("OV1.json")
    d = design_from_json(j)
    o = Oracle(d)
    b, nb = o.plan()
    seg, cost, dem = o.route(b, nb)
    viol, tot = o.overflow(seg, dem)
    assert list(viol) == j["expect"]["violating"]
    assert list(tot) == j["expect"]["totals"]


def test_tg1_hand_worked():
    j = load_golden("TG1.json")
    d = design_from_json(j)
    order, root, off, succ = Oracle(d).task_graph(np.arange(d.num_nets))
    e = j["expect"]
    assert list(order) == e["order"] and list(root) == e["is_root"]
    assert list(off) == e["succ_offset"] and list(succ) == e["succ"]


def _capacity(d, l, y, x):
    return int(d.edge_capacity[l, y, x]) if d.edge_capacity is not None else int(d.layer_capacity[l])


def py_overflow(d, seg, dem, zmid=None):
    """Independent recount: overflowed wire edges from the dense demand, violating nets from their legs."""
    cnt = tot = 0
    for l in range(d.nlayers):
        for y in range(d.ny):
            for x in range(d.nx):
                if (d.dir[l] == 0 and x == d.nx - 1) or (d.dir[l] == 1 and y == d.ny - 1):
                    continue
                over = int(dem[l, y, x]) - _capacity(d, l, y, x)
                if over > 0:
                    cnt += 1
                    tot += over
    viol = np.zeros(d.num_nets, np.uint8)
    for n in range(d.num_nets):
        a, b = d.node_offset[n], d.node_offset[n + 1]
        for v in range(a + 1, b):
            u = a + d.parent[v]
            z = -1 if zmid is None else int(zmid[v])
            for (l, xa, ya, xb, yb) in legs_of_edge(int(d.x[v]), int(d.y[v]), int(d.x[u]), int(d.y[u]), seg[v], z):
                cells = ([(ya, x) for x in range(min(xa, xb), max(xa, xb))] if ya == yb else
                         [(y, xa) for y in range(min(ya, yb), max(ya, yb))])
                if any(int(dem[l, y, x]) > _capacity(d, l, y, x) for y, x in cells):
                    viol[n] = 1
    return viol, (cnt, tot)


@pytest.mark.parametrize("seed,hybrid", [(0, None), (1, None), (2, (3, 40)), (3, (2, 60))])
def test_overflow_matches_recount(seed, hybrid):
    d = gen.random_small(seed=880 + seed, nx=30, ny=26, nlayers=4 + seed, num_nets=160, kmax=8,
                         literal_frac=0.3, caps=[1] * (4 + seed))
    o = Oracle(d)
    b, nb = o.plan()
    seg, cost, dem, zmid = o.route(b, nb, hybrid=hybrid, with_zmid=True)
    viol, tot = o.overflow(seg, dem, zmid)
    pv, pt = py_overflow(d, seg, dem, zmid)
    assert tot == pt and np.array_equal(viol, pv)
    assert tot[0] > 0 and 0 < viol.sum() < d.num_nets   # the case has both kinds of nets


def py_task_graph(d, tasks):
    keys = sorted((net_bbox(d, n)[2] - net_bbox(d, n)[0] + net_bbox(d, n)[3] - net_bbox(d, n)[1], n) for n in tasks)
    order = [n for _, n in keys]
    R = len(order)
    boxes = [net_bbox(d, n) for n in order]
    # root batch = colour 0 of first-fit colouring: no earlier conflicting task in colour 0
    root = []
    for i in range(R):
        root.append(not any(root[j] and boxes_touch(boxes[i], boxes[j]) for j in range(i)))
    succ = [[] for _ in range(R)]
    for i in range(R):
        for j in range(i + 1, R):
            if boxes_touch(boxes[i], boxes[j]):
                assert not (root[i] and root[j])
                if root[j]:
                    succ[j].append(i)
                else:
                    succ[i].append(j)
    off = [0]
    flat = []
    for s in succ:
        flat += sorted(s)
        off.append(len(flat))
    return order, root, off, flat


@pytest.mark.parametrize("seed", range(4))
def test_task_graph_bruteforce(seed):
    d = gen.random_small(seed=990 + seed, nx=40, ny=30, nlayers=4, num_nets=150, kmax=7, literal_frac=0.2)
    rng = np.random.default_rng(seed)
    tasks = np.sort(rng.choice(d.num_nets, 60, replace=False)).astype(np.int32)
    order, root, off, succ = Oracle(d).task_graph(tasks)
    po, pr, poff, psucc = py_task_graph(d, list(tasks))
    assert list(order) == po and [bool(x) for x in root] == pr
    assert list(off) == poff and list(succ) == psucc
    # the ordered graph is acyclic: roots have no predecessors, other edges go up in task ID
    for a in range(len(order)):
        for b in succ[off[a]:off[a + 1]]:
            assert root[a] or (not root[b] and a < b)
            assert not root[b]
