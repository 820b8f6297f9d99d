"""Python marshalling for the plain C oracle (oracle/fgr_oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this module.  It shares no
code with the CUDA path (paper_conf_date_liulzclly22_b200/).  What the oracle
computes, and the paper passages each step follows, is in the header of
oracle/fgr_oracle.c; parity status per function is in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

ORC_OK, ORC_INVALID, ORC_RANGE = 0, 1, 2


class _Grid(ctypes.Structure):
    _fields_ = [
        ("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nlayers", ctypes.c_int32),
        ("dir", ctypes.c_void_p), ("layer_capacity", ctypes.c_void_p), ("edge_capacity", ctypes.c_void_p),
        ("len_cost", ctypes.c_int32), ("via_cost", ctypes.c_void_p), ("ovf_weight", ctypes.c_void_p),
        ("logistic_slope", ctypes.c_double), ("slack_clamp", ctypes.c_int32),
    ]


class _Pattern(ctypes.Structure):
    _fields_ = [("hybrid_lo", ctypes.c_int32), ("hybrid_hi", ctypes.c_int32)]


def _pat(hybrid):
    """hybrid = None (L only) or (t1, t2): edges with t1 <= |dx|+|dy| <= t2 take hybrid L+Z patterns."""
    if hybrid is None:
        return None
    p = _Pattern()
    p.hybrid_lo, p.hybrid_hi = int(hybrid[0]), int(hybrid[1])
    return p


def _pp(p):
    return ctypes.byref(p) if p is not None else ctypes.c_void_p(0)


class _Nets(ctypes.Structure):
    _fields_ = [
        ("num_nets", ctypes.c_int32), ("node_offset", ctypes.c_void_p),
        ("x", ctypes.c_void_p), ("y", ctypes.c_void_p), ("pin_lo", ctypes.c_void_p),
        ("pin_hi", ctypes.c_void_p), ("parent", ctypes.c_void_p),
    ]


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(path)
        P = ctypes.c_void_p
        lib.orc_cost_table.argtypes = [P, P]
        lib.orc_validate.argtypes = [P, P, P]
        lib.orc_plan.argtypes = [P, P, P, P]
        lib.orc_route_net.argtypes = [P, P, ctypes.c_int32, P, P, P]
        lib.orc_commit_net.argtypes = [P, P, ctypes.c_int32, P, P]
        lib.orc_route.argtypes = [P, P, P, ctypes.c_int32, P, P, P, ctypes.c_int, P]
        lib.orc_recost_net.argtypes = [P, P, ctypes.c_int32, P, P, P]
        lib.orc_route_net_ex.argtypes = [P, P, ctypes.c_int32, P, P, P, P, P]
        lib.orc_commit_net_ex.argtypes = [P, P, ctypes.c_int32, P, P, P]
        lib.orc_route_ex.argtypes = [P, P, P, ctypes.c_int32, P, P, P, ctypes.c_int, P, P, P]
        lib.orc_recost_net_ex.argtypes = [P, P, ctypes.c_int32, P, P, P, P]
        lib.orc_overflow.argtypes = [P, P, P, P, P, P, P]
        lib.orc_task_graph.argtypes = [P, P, P, ctypes.c_int32, P, P, P, P, ctypes.c_int64, P]
        for f in ("orc_cost_table", "orc_validate", "orc_plan", "orc_route_net", "orc_commit_net",
                  "orc_route", "orc_recost_net", "orc_route_net_ex", "orc_commit_net_ex", "orc_route_ex",
                  "orc_recost_net_ex", "orc_overflow", "orc_task_graph"):
            getattr(lib, f).restype = ctypes.c_int
        _LIB = lib
    return _LIB


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else ctypes.c_void_p(0)


class Oracle:
    """Holds contiguous copies of one design so the C pointers stay valid."""

    def __init__(self, d):
        self.d = d
        self.L = d.nlayers
        self._keep = dict(
            dir=np.ascontiguousarray(d.dir, np.uint8),
            cap=np.ascontiguousarray(d.layer_capacity, np.int32),
            ecap=None if d.edge_capacity is None else np.ascontiguousarray(d.edge_capacity, np.uint8),
            via=np.ascontiguousarray(d.via_cost, np.int32),
            w=np.ascontiguousarray(d.ovf_weight, np.int32),
            off=np.ascontiguousarray(d.node_offset, np.int32),
            x=np.ascontiguousarray(d.x, np.int16), y=np.ascontiguousarray(d.y, np.int16),
            plo=np.ascontiguousarray(d.pin_lo, np.int8), phi=np.ascontiguousarray(d.pin_hi, np.int8),
            par=np.ascontiguousarray(d.parent, np.int32),
        )
        k = self._keep
        g = _Grid()
        g.nx, g.ny, g.nlayers = d.nx, d.ny, d.nlayers
        g.dir, g.layer_capacity = k["dir"].ctypes.data, k["cap"].ctypes.data
        g.edge_capacity = k["ecap"].ctypes.data if k["ecap"] is not None else None
        g.len_cost = d.len_cost
        g.via_cost, g.ovf_weight = k["via"].ctypes.data, k["w"].ctypes.data
        g.logistic_slope, g.slack_clamp = d.logistic_slope, d.slack_clamp
        n = _Nets()
        n.num_nets = d.num_nets
        n.node_offset = k["off"].ctypes.data
        n.x, n.y = k["x"].ctypes.data, k["y"].ctypes.data
        n.pin_lo, n.pin_hi, n.parent = k["plo"].ctypes.data, k["phi"].ctypes.data, k["par"].ctypes.data
        self.g, self.n = g, n

    # -- pieces -------------------------------------------------------------
    def cost_table(self) -> np.ndarray:
        S = self.d.slack_clamp
        t = np.zeros((self.L, 2 * S + 1), np.int64)
        _lib().orc_cost_table(ctypes.byref(self.g), _p(t))
        return t

    def validate(self):
        bad = np.zeros(1, np.int32)
        rc = _lib().orc_validate(ctypes.byref(self.g), ctypes.byref(self.n), _p(bad))
        return rc, int(bad[0])

    def zero_demand(self) -> np.ndarray:
        return np.zeros((self.L, self.d.ny, self.d.nx), np.int32)

    def plan(self):
        """Literal Algorithm 1 -> (batch_of_net int32[N] with -1 = trivial, num_batches)."""
        b = np.zeros(self.d.num_nets, np.int32)
        nb = np.zeros(1, np.int32)
        rc = _lib().orc_plan(ctypes.byref(self.g), ctypes.byref(self.n), _p(b), _p(nb))
        if rc != ORC_OK:
            raise ValueError(f"orc_plan rc={rc}")
        return b, int(nb[0])

    def route(self, batch_of_net, num_batches, demand=None, sequential=False, hashes=False, hybrid=None,
              with_zmid=False):
        """Batches in sequence -> (seg uint32[M], net_cost uint32[N], demand int32[L,ny,nx][, hashes][, zmid]).

        hybrid=(t1, t2) enables the hybrid L+Z patterns on edges with t1 <= |dx|+|dy| <= t2;
        zmid int32[M] = mid | lb << 16 for edges routed as a Z, -1 elsewhere."""
        dem = self.zero_demand() if demand is None else np.ascontiguousarray(demand, np.int32).copy()
        seg = np.zeros(self.d.num_nodes, np.uint32)
        cost = np.zeros(self.d.num_nets, np.uint32)
        zmid = np.full(self.d.num_nodes, -1, np.int32)
        bon = np.ascontiguousarray(batch_of_net, np.int32)
        h = np.zeros(max(num_batches, 1), np.uint64) if hashes else None
        pat = _pat(hybrid)
        rc = _lib().orc_route_ex(ctypes.byref(self.g), ctypes.byref(self.n), _p(bon), int(num_batches),
                                 _p(dem), _p(seg), _p(cost), int(bool(sequential)), _p(h), _pp(pat), _p(zmid))
        if rc != ORC_OK:
            raise ValueError(f"orc_route rc={rc}")
        out = [seg, cost, dem]
        if hashes:
            out.append(h[:num_batches])
        if with_zmid:
            out.append(zmid)
        return tuple(out)

    def route_net(self, net, demand, seg=None, hybrid=None, zmid=None):
        """One net's DP on a given demand; returns (seg uint32[M] with this net filled, cost)."""
        if seg is None:
            seg = np.zeros(self.d.num_nodes, np.uint32)
        dem = np.ascontiguousarray(demand, np.int32)
        c = np.zeros(1, np.uint32)
        rc = _lib().orc_route_net_ex(ctypes.byref(self.g), ctypes.byref(self.n), int(net), _p(dem), _p(seg), _p(c),
                                     _pp(_pat(hybrid)), _p(zmid))
        if rc != ORC_OK:
            raise ValueError(f"orc_route_net rc={rc}")
        return seg, int(c[0])

    def commit_net(self, net, seg, demand, zmid=None):
        _lib().orc_commit_net_ex(ctypes.byref(self.g), ctypes.byref(self.n), int(net),
                                 _p(np.ascontiguousarray(seg, np.uint32)),
                                 _p(None if zmid is None else np.ascontiguousarray(zmid, np.int32)), _p(demand))

    def recost_net(self, net, demand, seg, zmid=None) -> int:
        c = np.zeros(1, np.uint64)
        _lib().orc_recost_net_ex(ctypes.byref(self.g), ctypes.byref(self.n), int(net),
                                 _p(np.ascontiguousarray(demand, np.int32)),
                                 _p(np.ascontiguousarray(seg, np.uint32)),
                                 _p(None if zmid is None else np.ascontiguousarray(zmid, np.int32)), _p(c))
        return int(c[0])

    def overflow(self, seg, demand, zmid=None):
        """Rip-up set on a final demand -> (violating uint8[N], (overflowed edges, total overflow))."""
        viol = np.zeros(max(self.d.num_nets, 1), np.uint8)
        tot = np.zeros(2, np.int64)
        _lib().orc_overflow(ctypes.byref(self.g), ctypes.byref(self.n), _p(np.ascontiguousarray(seg, np.uint32)),
                            _p(None if zmid is None else np.ascontiguousarray(zmid, np.int32)),
                            _p(np.ascontiguousarray(demand, np.int32)), _p(viol), _p(tot))
        return viol[:self.d.num_nets], (int(tot[0]), int(tot[1]))

    def task_graph(self, tasks):
        """Ordered task graph of net ids `tasks` -> (order, is_root, succ_offset, succ) (task-ID indexed)."""
        tasks = np.ascontiguousarray(tasks, np.int32)
        R = len(tasks)
        order = np.zeros(max(R, 1), np.int32)
        root = np.zeros(max(R, 1), np.uint8)
        off = np.zeros(R + 1, np.int32)
        ne = np.zeros(1, np.int64)
        cap = 0
        while True:
            succ = np.zeros(max(cap, 1), np.int32)
            rc = _lib().orc_task_graph(ctypes.byref(self.g), ctypes.byref(self.n), _p(tasks), R, _p(order),
                                       _p(root), _p(off), _p(succ), int(cap), _p(ne))
            if rc == ORC_OK:
                return order[:R], root[:R], off, succ[:int(ne[0])]
            if rc != ORC_RANGE:
                raise ValueError(f"orc_task_graph rc={rc}")
            cap = int(ne[0])

    def run(self):
        """Whole stage: plan + route from zero demand."""
        b, nb = self.plan()
        seg, cost, dem = self.route(b, nb)
        return b, nb, seg, cost, dem
