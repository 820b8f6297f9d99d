"""Shared test helpers: golden-file designs, independent recounts and brute force.

Nothing here calls the CUDA path or the oracle's internals; these are the
independent checks the oracle is pinned against.
"""
import itertools
import json
import math
import os

import numpy as np

from gen import Design

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def design_from_json(j) -> Design:
    L, nx, ny = j["nlayers"], j["nx"], j["ny"]
    xs, ys, plo, phi, par, off = [], [], [], [], [], [0]
    for n in j["nets"]:
        xs += n["x"]; ys += n["y"]; plo += n["pin_lo"]; phi += n["pin_hi"]; par += n["parent"]
        off.append(off[-1] + len(n["x"]))
    ecap = None
    if "edge_capacity_override" in j:
        ecap = np.empty((L, ny, nx), np.uint8)
        for l in range(L):
            ecap[l] = j["layer_capacity"][l]
        for l, y, x, c in j["edge_capacity_override"]:
            ecap[l, y, x] = c
    d = Design(nx, ny, L, np.array(j["dir"], np.uint8), np.array(j["layer_capacity"], np.int32), ecap,
               np.array(off, np.int32), np.array(xs, np.int16), np.array(ys, np.int16),
               np.array(plo, np.int8), np.array(phi, np.int8), np.array(par, np.int32),
               name=j["name"], len_cost=j["len_cost"], via_cost=np.array(j["via_cost"], np.int32),
               ovf_weight=np.array(j["ovf_weight"], np.int32), logistic_slope=j["logistic_slope"],
               slack_clamp=j["slack_clamp"])
    return d


def seg_fields(s):
    s = int(s)
    return dict(bend=s & 0xFF, ls=(s >> 8) & 0xFF, lt=(s >> 16) & 0xFF, straight=(s >> 24) & 0xFF)


def make_seg(bend, ls, lt, straight):
    return bend | (ls << 8) | (lt << 16) | (straight << 24)


def legs_of_edge(xv, yv, xu, yu, seg, z=-1):
    """[(layer, xa, ya, xb, yb)] of a chosen route for tree edge v -> u (include/fastgr.h semantics).

    bend 2 / 3 = Z shape HVH / VHV (§III-E) with z = mid | lb << 16."""
    f = seg_fields(seg)
    if f["straight"]:
        return [(f["lt"], xv, yv, xu, yu)]
    if f["bend"] >= 2:
        mid, lb = z & 0xFFFF, (z >> 16) & 0xFF
        if f["bend"] == 2:
            bs, bt = (mid, yv), (mid, yu)
        else:
            bs, bt = (xv, mid), (xu, mid)
        return [(f["ls"], xv, yv) + bs, (lb,) + bs + bt, (f["lt"],) + bt + (xu, yu)]
    if f["bend"] == 0:
        bx, by = xu, yv
    else:
        bx, by = xv, yu
    return [(f["ls"], xv, yv, bx, by), (f["lt"], bx, by, xu, yu)]


def recount_demand(d: Design, seg, base=None, zmid=None):
    """Demand = base + sum over committed legs (independent recount from seg)."""
    dem = np.zeros((d.nlayers, d.ny, d.nx), np.int64) if base is None else base.astype(np.int64).copy()
    for n in range(d.num_nets):
        a, b = d.node_offset[n], d.node_offset[n + 1]
        for v in range(a + 1, b):
            u = a + d.parent[v]
            z = -1 if zmid is None else int(zmid[v])
            for (l, xa, ya, xb, yb) in legs_of_edge(int(d.x[v]), int(d.y[v]), int(d.x[u]), int(d.y[u]), seg[v], z):
                if ya == yb:
                    for x in range(min(xa, xb), max(xa, xb)):
                        dem[l, ya, x] += 1
                else:
                    for y in range(min(ya, yb), max(ya, yb)):
                        dem[l, y, xa] += 1
    return dem


def net_bbox(d: Design, n):
    a, b = d.node_offset[n], d.node_offset[n + 1]
    return (int(d.x[a:b].min()), int(d.y[a:b].min()), int(d.x[a:b].max()), int(d.y[a:b].max()))


def boxes_touch(b1, b2):
    return not (b1[2] < b2[0] or b2[2] < b1[0] or b1[3] < b2[1] or b2[3] < b1[1])


def sort_order(d: Design):
    """Non-trivial nets by (HPWL, id) — the order Algorithm 1 consumes (reading R12)."""
    keys = []
    for n in range(d.num_nets):
        if d.node_offset[n + 1] - d.node_offset[n] < 2:
            continue
        x0, y0, x1, y1 = net_bbox(d, n)
        keys.append((x1 - x0 + y1 - y0, n))
    keys.sort()
    return [n for _, n in keys]


# ---------------------------------------------------------------- brute force
def logistic_table_py(W, slope, S):
    """Round-half-away of W/(1+exp(slope*s)); used only by the brute force."""
    out = {}
    for s in range(-S, S + 1):
        v = W / (1.0 + math.exp(slope * s))
        out[s] = int(math.floor(v + 0.5))
    return out


class PyCost:
    """Per-edge costs straight from the definition, for brute-force enumeration."""

    def __init__(self, d: Design, demand):
        self.d = d
        self.dem = demand
        self.tab = [logistic_table_py(int(d.ovf_weight[l]), d.logistic_slope, d.slack_clamp) for l in range(d.nlayers)]

    def cap(self, l, y, x):
        if self.d.edge_capacity is not None:
            return int(self.d.edge_capacity[l, y, x])
        return int(self.d.layer_capacity[l])

    def ec(self, l, y, x):
        S = self.d.slack_clamp
        s = max(-S, min(S, self.cap(l, y, x) - int(self.dem[l, y, x])))
        return self.d.len_cost + self.tab[l][s]

    def wire(self, l, xa, ya, xb, yb):
        if xa == xb and ya == yb:
            return 0
        if ya == yb:
            if self.d.dir[l] != 0:
                return None
            return sum(self.ec(l, ya, x) for x in range(min(xa, xb), max(xa, xb)))
        if self.d.dir[l] != 1:
            return None
        return sum(self.ec(l, y, xa) for y in range(min(ya, yb), max(ya, yb)))

    def via(self, a, b):
        lo, hi = min(a, b), max(a, b)
        return int(sum(int(self.d.via_cost[k]) for k in range(lo, hi)))


def route_cost(d: Design, pc: PyCost, n, segs, zs=None):
    """Cost of a complete assignment: wires + bend-point vias + node via hulls (None if illegal).

    segs[i] / zs[i] = the route of local node i's edge (zs: Z middle, see legs_of_edge)."""
    a, b = d.node_offset[n], d.node_offset[n + 1]
    m = b - a
    L = d.nlayers
    lo = [int(d.pin_lo[a + i]) if d.pin_lo[a + i] >= 0 else L for i in range(m)]
    hi = [int(d.pin_hi[a + i]) if d.pin_hi[a + i] >= 0 else -1 for i in range(m)]
    total = 0
    for i in range(1, m):
        v, u = a + i, a + int(d.parent[a + i])
        f = seg_fields(segs[i])
        legs = legs_of_edge(int(d.x[v]), int(d.y[v]), int(d.x[u]), int(d.y[u]), segs[i],
                            -1 if zs is None else zs[i])
        for k, (l, xa, ya, xb, yb) in enumerate(legs):
            w = pc.wire(l, xa, ya, xb, yb)
            if w is None:
                return None
            total += w
            if k > 0:
                total += pc.via(legs[k - 1][0], l)
        ui = int(d.parent[a + i])
        lo[i] = min(lo[i], f["ls"]); hi[i] = max(hi[i], f["ls"])
        lo[ui] = min(lo[ui], f["lt"]); hi[ui] = max(hi[ui], f["lt"])
    for i in range(m):
        if hi[i] >= lo[i]:
            total += pc.via(lo[i], hi[i])
    return total


def edge_options(d: Design, n, i, hybrid=None, general_straight=False):
    """Every route of local node i's edge: [(seg, z)].  With hybrid=(t1, t2) and t1 <= HPWL <= t2
    (bent edges only), every Z shape with both bend points strictly inside the box is added.

    general_straight=True (the check of reading R7): a straight edge also gets both degenerate
    L shapes with any layer pair — one leg along the edge on a layer of its direction, a
    zero-length leg on ANY layer at an endpoint, and the bend via between the two (so the
    via stack at that endpoint may be paid at the "bend" instead of in the node hull)."""
    a = d.node_offset[n]
    v, u = a + i, a + int(d.parent[a + i])
    xv, yv, xu, yu = int(d.x[v]), int(d.y[v]), int(d.x[u]), int(d.y[u])
    L = d.nlayers
    H = [l for l in range(L) if d.dir[l] == 0]
    V = [l for l in range(L) if d.dir[l] == 1]
    if yv == yu or xv == xu:
        D = H if yv == yu else V
        out = [(make_seg(0, l, l, 1), -1) for l in D]
        if general_straight:
            # bend 0 (bend point (x_u, y_v)) and bend 1 (bend point (x_v, y_u)); for a horizontal edge
            # bend 0 = full leg 1 on ls in H then zero-length leg 2 at u on any lt, bend 1 = zero-length
            # leg 1 at v on any ls then full leg 2 on lt in H (vertical edges: the mirror image)
            full_first = 0 if yv == yu else 1
            out += [(make_seg(full_first, ls, lt, 0), -1) for ls in D for lt in range(L) if lt != ls]
            out += [(make_seg(1 - full_first, ls, lt, 0), -1) for lt in D for ls in range(L) if ls != lt]
        return out
    out = [(make_seg(0, ls, lt, 0), -1) for ls in H for lt in V] + [(make_seg(1, ls, lt, 0), -1) for ls in V for lt in H]
    h = abs(xv - xu) + abs(yv - yu)
    if hybrid is not None and hybrid[0] <= h <= hybrid[1]:
        for xm in range(min(xv, xu) + 1, max(xv, xu)):
            out += [(make_seg(2, ls, lt, 0), xm | (lb << 16)) for ls in H for lb in V for lt in H]
        for ym in range(min(yv, yu) + 1, max(yv, yu)):
            out += [(make_seg(3, ls, lt, 0), ym | (lb << 16)) for ls in V for lb in H for lt in V]
    return out


def brute_force_min(d: Design, n, demand, hybrid=None, general_straight=False):
    """Min over every per-edge route assignment of the full route cost."""
    pc = PyCost(d, demand)
    m = d.node_offset[n + 1] - d.node_offset[n]
    opts = [edge_options(d, n, i, hybrid, general_straight) for i in range(1, m)]
    best = None
    for combo in itertools.product(*opts):
        c = route_cost(d, pc, n, [None] + [s for s, _ in combo], [None] + [z for _, z in combo])
        if c is not None and (best is None or c < best):
            best = c
    return best
