"""Seeded synthetic design generator (shared input plumbing; no method arithmetic).

Both the CUDA path (tests, bench) and the oracle take their inputs from here.
The heavy lifting is in ``gen/fgr_gen.c`` (compiled to ``gen/libfgrgen.so`` by
``make``); this module only marshals parameters and copies the result into
numpy arrays.  The recipe (pin-count mix, lognormal HPWL, hotspots, congested
core, Prim MST + one median-Steiner pass) is stated in DESIGN.md §4 and follows
SURVEY.md §8(d).  Paper passages for the input *shape*: nets are pin point sets
mapped onto G-cells given as trees of two-pin nets
(L227-233); one preferred direction per layer (L203-206).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


class _Params(ctypes.Structure):
    _fields_ = [
        ("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nlayers", ctypes.c_int32),
        ("num_nets", ctypes.c_int32), ("seed", ctypes.c_uint64),
        ("layer_capacity", ctypes.c_int32 * 16),
        ("pin_dist", ctypes.c_int32), ("kmin", ctypes.c_int32), ("kmax", ctypes.c_int32),
        ("hpwl_sigma", ctypes.c_double), ("hpwl_base", ctypes.c_double),
        ("literal_frac", ctypes.c_double),
        ("hotspots", ctypes.c_int32), ("hot_frac", ctypes.c_double), ("hot_sigma_frac", ctypes.c_double),
        ("congested_core", ctypes.c_int32), ("steiner", ctypes.c_int32),
    ]


class _Design(ctypes.Structure):
    _fields_ = [
        ("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nlayers", ctypes.c_int32),
        ("dir", ctypes.c_uint8 * 16), ("layer_capacity", ctypes.c_int32 * 16),
        ("edge_capacity", ctypes.POINTER(ctypes.c_uint8)),
        ("num_nets", ctypes.c_int32), ("num_nodes", ctypes.c_int32),
        ("node_offset", ctypes.POINTER(ctypes.c_int32)),
        ("x", ctypes.POINTER(ctypes.c_int16)), ("y", ctypes.POINTER(ctypes.c_int16)),
        ("pin_lo", ctypes.POINTER(ctypes.c_int8)), ("pin_hi", ctypes.POINTER(ctypes.c_int8)),
        ("parent", ctypes.POINTER(ctypes.c_int32)),
        ("cap_nodes", ctypes.c_int64),
    ]


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libfgrgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make` (or __graft_entry__.build())")
        _LIB = ctypes.CDLL(path)
        _LIB.fgr_gen_design.argtypes = [ctypes.POINTER(_Params), ctypes.POINTER(_Design)]
        _LIB.fgr_gen_design.restype = ctypes.c_int
        _LIB.fgr_gen_free.argtypes = [ctypes.POINTER(_Design)]
        _LIB.fgr_gen_free.restype = None
    return _LIB


@dataclass
class Design:
    """A grid plus nets, all host numpy arrays (layouts documented in include/fastgr.h)."""
    nx: int
    ny: int
    nlayers: int
    dir: np.ndarray              # uint8 [L], 0 = H, 1 = V
    layer_capacity: np.ndarray   # int32 [L]
    edge_capacity: Optional[np.ndarray]  # uint8 [L, ny, nx] or None
    node_offset: np.ndarray      # int32 [N+1]
    x: np.ndarray                # int16 [M]
    y: np.ndarray                # int16 [M]
    pin_lo: np.ndarray           # int8 [M]
    pin_hi: np.ndarray           # int8 [M]
    parent: np.ndarray           # int32 [M] net-local, parent[i] < i, -1 at local 0
    name: str = ""
    seed: int = 0
    # cost parameters (defaults: DESIGN.md reading R1/R2)
    len_cost: int = 64
    via_cost: np.ndarray = field(default=None)      # int32 [L-1]
    ovf_weight: np.ndarray = field(default=None)    # int32 [L]
    logistic_slope: float = 1.0
    slack_clamp: int = 64

    def __post_init__(self):
        if self.via_cost is None:
            self.via_cost = np.full(self.nlayers - 1, 32, np.int32)
        if self.ovf_weight is None:
            self.ovf_weight = np.full(self.nlayers, 4096, np.int32)

    @property
    def num_nets(self) -> int:
        return len(self.node_offset) - 1

    @property
    def num_nodes(self) -> int:
        return int(self.node_offset[-1])

    def net_sizes(self) -> np.ndarray:
        return np.diff(self.node_offset)

    def subset(self, net_ids) -> "Design":
        """A design with only the given nets (same grid); used for bounded samples."""
        net_ids = np.asarray(net_ids, np.int64)
        sizes = self.net_sizes()[net_ids]
        off = np.zeros(len(net_ids) + 1, np.int32)
        np.cumsum(sizes, out=off[1:])
        idx = np.concatenate([np.arange(self.node_offset[i], self.node_offset[i + 1]) for i in net_ids]) \
            if len(net_ids) else np.zeros(0, np.int64)
        return Design(self.nx, self.ny, self.nlayers, self.dir.copy(), self.layer_capacity.copy(),
                      None if self.edge_capacity is None else self.edge_capacity.copy(),
                      off, self.x[idx].copy(), self.y[idx].copy(), self.pin_lo[idx].copy(),
                      self.pin_hi[idx].copy(), self.parent[idx].copy(), name=self.name + "-subset",
                      seed=self.seed, len_cost=self.len_cost, via_cost=self.via_cost.copy(),
                      ovf_weight=self.ovf_weight.copy(), logistic_slope=self.logistic_slope,
                      slack_clamp=self.slack_clamp)


# SURVEY.md §8(d) configs.  L=9 capacities: layer 0 is the low-capacity M1-like pin layer.
CAP9 = [2, 10, 10, 10, 10, 10, 10, 8, 8]
CONFIGS = {
    # tiny: 64x64/5, 200 nets of 2-6 pins, half paper-literal, tight capacity (so congestion matters)
    "tiny": dict(nx=64, ny=64, nlayers=5, num_nets=200, seed=1, caps=[1, 2, 2, 2, 2], pin_dist=1,
                 kmin=2, kmax=6, hpwl_base=6.0, hpwl_sigma=0.6, literal_frac=0.5, hotspots=1,
                 hot_frac=0.5, hot_sigma_frac=0.15, congested_core=0),
    "t1": dict(nx=200, ny=200, nlayers=9, num_nets=3000, seed=18001, caps=CAP9, pin_dist=0,
               hpwl_base=3.0, hpwl_sigma=0.7, literal_frac=0.0, hotspots=0, hot_frac=0.0,
               hot_sigma_frac=0.1, congested_core=0),
    "t5": dict(nx=300, ny=300, nlayers=9, num_nets=72000, seed=18005, caps=CAP9, pin_dist=0,
               hpwl_base=3.0, hpwl_sigma=0.7, literal_frac=0.0, hotspots=0, hot_frac=0.0,
               hot_sigma_frac=0.1, congested_core=1),
    "t9": dict(nx=900, ny=900, nlayers=9, num_nets=900000, seed=19009, caps=CAP9, pin_dist=0,
               hpwl_base=3.0, hpwl_sigma=0.7, literal_frac=0.0, hotspots=4, hot_frac=0.2,
               hot_sigma_frac=0.1, congested_core=0),
    "scale": dict(nx=2000, ny=2000, nlayers=9, num_nets=2000000, seed=2000, caps=CAP9, pin_dist=0,
                  hpwl_base=3.0, hpwl_sigma=0.7, literal_frac=0.0, hotspots=4, hot_frac=0.2,
                  hot_sigma_frac=0.1, congested_core=0),
}


def generate(nx, ny, nlayers, num_nets, seed, caps, pin_dist=0, kmin=2, kmax=6, hpwl_base=3.0,
             hpwl_sigma=0.7, literal_frac=0.0, hotspots=0, hot_frac=0.0, hot_sigma_frac=0.1,
             congested_core=0, steiner=1, name="custom") -> Design:
    p = _Params()
    p.nx, p.ny, p.nlayers, p.num_nets, p.seed = nx, ny, nlayers, num_nets, seed
    for i, c in enumerate(caps):
        p.layer_capacity[i] = c
    p.pin_dist, p.kmin, p.kmax = pin_dist, kmin, kmax
    p.hpwl_sigma, p.hpwl_base, p.literal_frac = hpwl_sigma, hpwl_base, literal_frac
    p.hotspots, p.hot_frac, p.hot_sigma_frac = hotspots, hot_frac, hot_sigma_frac
    p.congested_core, p.steiner = congested_core, steiner
    d = _Design()
    lib = _lib()
    if lib.fgr_gen_design(ctypes.byref(p), ctypes.byref(d)) != 0:
        raise ValueError("bad generator parameters")
    try:
        N, M = d.num_nets, d.num_nodes

        def arr(ptr, n, dt):
            if n == 0:
                return np.zeros(0, dt)
            return np.ctypeslib.as_array(ptr, shape=(n,)).astype(dt, copy=True)

        ecap = None
        if d.edge_capacity:
            ecap = arr(d.edge_capacity, nlayers * nx * ny, np.uint8).reshape(nlayers, ny, nx)
        out = Design(nx, ny, nlayers, np.array(d.dir[:nlayers], np.uint8),
                     np.array(d.layer_capacity[:nlayers], np.int32), ecap,
                     arr(d.node_offset, N + 1, np.int32), arr(d.x, M, np.int16), arr(d.y, M, np.int16),
                     arr(d.pin_lo, M, np.int8), arr(d.pin_hi, M, np.int8), arr(d.parent, M, np.int32),
                     name=name, seed=seed)
    finally:
        lib.fgr_gen_free(ctypes.byref(d))
    return out


def make_config(name: str, num_nets: Optional[int] = None, seed: Optional[int] = None) -> Design:
    c = dict(CONFIGS[name])
    caps = c.pop("caps")
    if num_nets is not None:
        c["num_nets"] = num_nets
    if seed is not None:
        c["seed"] = seed
    return generate(caps=caps, name=name, **c)


def random_small(seed: int, nx=12, ny=10, nlayers=4, num_nets=20, kmax=5, literal_frac=0.3,
                 caps=None, congested_core=0) -> Design:
    """Small random designs for fuzz/parity tests."""
    if caps is None:
        caps = [1] + [2] * (nlayers - 1)
    return generate(nx=nx, ny=ny, nlayers=nlayers, num_nets=num_nets, seed=seed, caps=caps,
                    pin_dist=1, kmin=2, kmax=kmax, hpwl_base=3.0, hpwl_sigma=0.6,
                    literal_frac=literal_frac, congested_core=congested_core, name=f"rand{seed}")
