"""Thin ctypes binding of libfastgr (include/fastgr.h): argument marshalling only.

Every step of the path runs in the library's CUDA kernels; this module only
packs structs, passes device pointers (torch tensors are used for device memory
and streams) and turns status codes into exceptions.  There is no CPU fallback:
importing works without a GPU (so the ABI can be checked on CPU), but every
compute call needs the CUDA library and a device, and fails loudly otherwise.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FGR_LIB_PATH") or os.path.join(_HERE, "libfastgr.so")
_LIB = None

FGR_OK, FGR_ERR_INVALID, FGR_ERR_RANGE, FGR_ERR_OOM, FGR_ERR_CUDA, FGR_ERR_NCCL, FGR_ERR_STATE = range(7)
FGR_DP_AUTO, FGR_DP_HEAVY, FGR_DP_HLD = 0, 1, 2   # large-net DP kernel selection (fgr_set_dp_policy)
STATUS_NAMES = ["OK", "INVALID", "RANGE", "OOM", "CUDA", "NCCL", "STATE"]

# every entry point include/fastgr.h declares
EXPORTS = ["fgr_last_error", "fgr_version", "fgr_cost_table", "fgr_grid_create", "fgr_grid_destroy",
           "fgr_grid_set_demand", "fgr_grid_get_demand", "fgr_plan", "fgr_route_batch", "fgr_route_all",
           "fgr_comm_unique_id", "fgr_comm_init", "fgr_run_host", "fgr_get_stats", "fgr_profile_enable",
           "fgr_profile_read", "fgr_split_batch", "fgr_set_pattern", "fgr_route_batch_ex", "fgr_route_all_ex",
           "fgr_run_host_ex", "fgr_overflow", "fgr_task_graph", "fgr_set_dp_policy", "fgr_set_exchange", "fgr_set_graph"]
PROF_CLASSES = ["refresh", "dp_small", "dp_large", "commit", "plan_preprocess", "plan_sort", "plan_color",
                "plan_other", "exchange", "hybrid"]
# the paper's FastGRH selection window: hybrid L+Z on two-pin HPWL in [100, 500]
HYBRID_PAPER = (100, 500)


class FgrError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"FGR_ERR_{STATUS_NAMES[status] if 0 <= status < 7 else status}: {msg}")
        self.status = status


class fgr_grid_desc(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nlayers", ctypes.c_int32),
                ("dir", ctypes.c_void_p), ("layer_capacity", ctypes.c_void_p), ("edge_capacity", ctypes.c_void_p),
                ("len_cost", ctypes.c_int32), ("via_cost", ctypes.c_void_p), ("ovf_weight", ctypes.c_void_p),
                ("logistic_slope", ctypes.c_double), ("slack_clamp", ctypes.c_int32)]


class fgr_nets(ctypes.Structure):
    _fields_ = [("num_nets", ctypes.c_int32), ("num_nodes", ctypes.c_int32), ("node_offset", ctypes.c_void_p),
                ("x", ctypes.c_void_p), ("y", ctypes.c_void_p), ("pin_lo", ctypes.c_void_p),
                ("pin_hi", ctypes.c_void_p), ("parent", ctypes.c_void_p)]


class fgr_stats(ctypes.Structure):
    _fields_ = [("refresh_segments", ctypes.c_int64), ("refresh_bytes", ctypes.c_int64), ("dp_nets", ctypes.c_int64),
                ("dp_edges", ctypes.c_int64), ("kernel_launches", ctypes.c_int64), ("num_batches", ctypes.c_int32),
                ("world", ctypes.c_int32), ("rank", ctypes.c_int32), ("exchanged_batches", ctypes.c_int32),
                ("graph_mode", ctypes.c_int32), ("reserved", ctypes.c_int32)]


def lib():
    """Load libfastgr.so (built in-tree by `make` / __graft_entry__.build())."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: the CUDA extension must be built (make); "
                               "there is no fallback path")
        L = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
        P, I, S = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int
        sig = {
            "fgr_last_error": ([], ctypes.c_char_p),
            "fgr_version": ([], ctypes.c_char_p),
            "fgr_cost_table": ([P, P], S),
            "fgr_grid_create": ([P, S, P, P], S),
            "fgr_grid_destroy": ([P], S),
            "fgr_grid_set_demand": ([P, P, P], S),
            "fgr_grid_get_demand": ([P, P, P], S),
            "fgr_plan": ([P, P, P, P, P, P, P], S),
            "fgr_route_batch": ([P, P, P, I, P, P, P], S),
            "fgr_route_all": ([P, P, P, P, I, P, P, P], S),
            "fgr_comm_unique_id": ([P], S),
            "fgr_comm_init": ([P, P, S, S], S),
            "fgr_run_host": ([P, I, I, P, P, P, P, P, P, P, P, P, P], S),
            "fgr_get_stats": ([P, P], S),
            "fgr_profile_enable": ([P, S], S),
            "fgr_profile_read": ([P, P, P], S),
            "fgr_split_batch": ([I, I, P, I, I, I, P], S),
            "fgr_set_exchange": ([P, I, I], S),
            "fgr_set_graph": ([P, I], S),
            "fgr_set_pattern": ([P, I, I], S),
            "fgr_set_dp_policy": ([P, I, I], S),
            "fgr_route_batch_ex": ([P, P, P, I, P, P, P, P], S),
            "fgr_route_all_ex": ([P, P, P, P, I, P, P, P, P], S),
            "fgr_run_host_ex": ([P, I, I, P, P, P, P, P, P, P, P, P, P, P], S),
            "fgr_overflow": ([P, P, P, P, P, P, P, P, P], S),
            "fgr_task_graph": ([P, P, P, I, P, P, P, P, ctypes.c_int64, P, P], S),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes, f.restype = args, res
        _LIB = L
    return _LIB


def _check(status):
    if status != FGR_OK:
        raise FgrError(status, lib().fgr_last_error().decode())


def _ptr(t):
    """Device/host address of a torch tensor or numpy array (None -> NULL)."""
    if t is None:
        return None
    if isinstance(t, np.ndarray):
        return t.ctypes.data
    return t.data_ptr()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return stream if isinstance(stream, int) else stream.cuda_stream


# ----------------------------------------------------------------- C names
def fgr_version() -> str:
    return lib().fgr_version().decode()


def make_desc(nx, ny, nlayers, dir, layer_capacity, len_cost, via_cost, ovf_weight, logistic_slope, slack_clamp,
              edge_capacity_dev=None):
    keep = [np.ascontiguousarray(dir, np.uint8), np.ascontiguousarray(layer_capacity, np.int32),
            np.ascontiguousarray(via_cost, np.int32), np.ascontiguousarray(ovf_weight, np.int32)]
    d = fgr_grid_desc(nx, ny, nlayers, keep[0].ctypes.data, keep[1].ctypes.data, _ptr(edge_capacity_dev), len_cost,
                      keep[2].ctypes.data, keep[3].ctypes.data, float(logistic_slope), slack_clamp)
    d._keep = keep
    return d


def fgr_cost_table(desc) -> np.ndarray:
    t = np.zeros((desc.nlayers, 2 * desc.slack_clamp + 1), np.int64)
    _check(lib().fgr_cost_table(ctypes.byref(desc), t.ctypes.data))
    return t


def fgr_grid_create(desc, device=0, stream=None):
    h = ctypes.c_void_p()
    _check(lib().fgr_grid_create(ctypes.byref(desc), device, _stream(stream), ctypes.byref(h)))
    return h


def fgr_grid_destroy(h):
    _check(lib().fgr_grid_destroy(h))


def fgr_grid_set_demand(h, demand=None, stream=None):
    _check(lib().fgr_grid_set_demand(h, _ptr(demand), _stream(stream)))


def fgr_grid_get_demand(h, out, stream=None):
    _check(lib().fgr_grid_get_demand(h, _ptr(out), _stream(stream)))


def make_nets(num_nets, num_nodes, node_offset, x, y, pin_lo, pin_hi, parent):
    n = fgr_nets(num_nets, num_nodes, _ptr(node_offset), _ptr(x), _ptr(y), _ptr(pin_lo), _ptr(pin_hi), _ptr(parent))
    n._keep = (node_offset, x, y, pin_lo, pin_hi, parent)
    return n


def fgr_plan(h, nets, batch_of_net, order, batch_offset, stream=None) -> int:
    nb = ctypes.c_int32(0)
    _check(lib().fgr_plan(h, ctypes.byref(nets), _ptr(batch_of_net), _ptr(order), _ptr(batch_offset),
                          ctypes.byref(nb), _stream(stream)))
    return nb.value


def fgr_route_batch(h, nets, net_ids, count, seg_out, net_cost, stream=None):
    _check(lib().fgr_route_batch(h, ctypes.byref(nets), _ptr(net_ids), int(count), _ptr(seg_out), _ptr(net_cost),
                                 _stream(stream)))


def fgr_route_all(h, nets, order, batch_offset, num_batches, seg_out, net_cost, stream=None):
    _check(lib().fgr_route_all(h, ctypes.byref(nets), _ptr(order), _ptr(batch_offset), int(num_batches),
                               _ptr(seg_out), _ptr(net_cost), _stream(stream)))


def fgr_set_pattern(h, hybrid_t1, hybrid_t2):
    _check(lib().fgr_set_pattern(h, int(hybrid_t1), int(hybrid_t2)))


def fgr_set_dp_policy(h, policy, flow_max=64):
    _check(lib().fgr_set_dp_policy(h, int(policy), int(flow_max)))


def fgr_route_batch_ex(h, nets, net_ids, count, seg_out, zmid_out, net_cost, stream=None):
    _check(lib().fgr_route_batch_ex(h, ctypes.byref(nets), _ptr(net_ids), int(count), _ptr(seg_out), _ptr(zmid_out),
                                    _ptr(net_cost), _stream(stream)))


def fgr_route_all_ex(h, nets, order, batch_offset, num_batches, seg_out, zmid_out, net_cost, stream=None):
    _check(lib().fgr_route_all_ex(h, ctypes.byref(nets), _ptr(order), _ptr(batch_offset), int(num_batches),
                                  _ptr(seg_out), _ptr(zmid_out), _ptr(net_cost), _stream(stream)))


def fgr_comm_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().fgr_comm_unique_id(buf))
    return buf.raw


def fgr_comm_init(h, unique_id: bytes, rank: int, world: int):
    buf = ctypes.create_string_buffer(bytes(unique_id), 128)
    _check(lib().fgr_comm_init(h, buf, rank, world))


def fgr_run_host(h, node_offset, x, y, pin_lo, pin_hi, parent, seg_out=None, net_cost=None, stream=None) -> int:
    """Host-buffer end-to-end call (numpy or pinned CPU torch tensors)."""
    nb = ctypes.c_int32(0)
    N = len(node_offset) - 1
    M = len(x)
    _check(lib().fgr_run_host(h, N, M, _ptr(node_offset), _ptr(x), _ptr(y), _ptr(pin_lo), _ptr(pin_hi),
                              _ptr(parent), _ptr(seg_out), _ptr(net_cost), ctypes.byref(nb), _stream(stream)))
    return nb.value


def fgr_run_host_ex(h, node_offset, x, y, pin_lo, pin_hi, parent, seg_out=None, zmid_out=None, net_cost=None,
                    stream=None) -> int:
    nb = ctypes.c_int32(0)
    N = len(node_offset) - 1
    M = len(x)
    _check(lib().fgr_run_host_ex(h, N, M, _ptr(node_offset), _ptr(x), _ptr(y), _ptr(pin_lo), _ptr(pin_hi),
                                 _ptr(parent), _ptr(seg_out), _ptr(zmid_out), _ptr(net_cost), ctypes.byref(nb),
                                 _stream(stream)))
    return nb.value


def fgr_overflow(h, nets, seg, zmid, violating, rip_ids, stream=None):
    """-> (num_rip, (overflowed edges, total overflow)); violating / rip_ids filled on the device."""
    nr = ctypes.c_int32(0)
    tot = np.zeros(2, np.int64)
    _check(lib().fgr_overflow(h, ctypes.byref(nets), _ptr(seg), _ptr(zmid), _ptr(violating), _ptr(rip_ids),
                              ctypes.byref(nr), tot.ctypes.data, _stream(stream)))
    return nr.value, (int(tot[0]), int(tot[1]))


def fgr_task_graph(h, nets, tasks, count, order, is_root, succ_offset, succ, capacity, stream=None) -> int:
    """-> number of directed edges (raises FGR_ERR_RANGE when it exceeds capacity)."""
    ne = ctypes.c_int64(0)
    _check(lib().fgr_task_graph(h, ctypes.byref(nets), _ptr(tasks), int(count), _ptr(order), _ptr(is_root),
                                _ptr(succ_offset), _ptr(succ), int(capacity), ctypes.byref(ne), _stream(stream)))
    return ne.value


def fgr_get_stats(h) -> dict:
    s = fgr_stats()
    _check(lib().fgr_get_stats(h, ctypes.byref(s)))
    return {k: getattr(s, k) for k, _ in fgr_stats._fields_}


def fgr_split_batch(count, nlarge, rank, world, edge_prefix=None, split_min=0):
    """(large_lo, large_hi, small_lo, small_hi, whole) of `rank` for one batch (host-only)."""
    out = np.zeros(5, np.int32)
    ep = None if edge_prefix is None else np.ascontiguousarray(edge_prefix, np.int64)
    _check(lib().fgr_split_batch(int(count), int(nlarge), None if ep is None else ep.ctypes.data, int(split_min),
                                 int(rank), int(world), out.ctypes.data))
    return tuple(int(v) for v in out)


def fgr_set_exchange(h, split_min=2048, emulate_world=0):
    _check(lib().fgr_set_exchange(h, int(split_min), int(emulate_world)))


def fgr_set_graph(h, on=True):
    """Replay the single-GPU batch loop as a CUDA Graph (default on); routes are identical either way."""
    _check(lib().fgr_set_graph(h, 1 if on else 0))


def fgr_profile_enable(h, enable=True):
    _check(lib().fgr_profile_enable(h, 1 if enable else 0))


def fgr_profile_read(h) -> dict:
    ms = np.zeros(len(PROF_CLASSES), np.float64)
    n = np.zeros(len(PROF_CLASSES), np.int64)
    _check(lib().fgr_profile_read(h, ms.ctypes.data, n.ctypes.data))
    return {c: (float(ms[i]), int(n[i])) for i, c in enumerate(PROF_CLASSES)}


# ----------------------------------------------------------------- conveniences (marshalling only)
class Router:
    """Owns a grid handle plus device copies of one design's nets (torch tensors)."""

    def __init__(self, design, device: int = 0, stream=None, hybrid=None, dp_policy=None):
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError("fastgr needs a CUDA device (no CPU fallback)")
        self.torch = torch
        self.dev = torch.device("cuda", device)
        self.d = design
        ecap = None
        if design.edge_capacity is not None:
            ecap = torch.from_numpy(np.ascontiguousarray(design.edge_capacity)).to(self.dev)
        self.desc = make_desc(design.nx, design.ny, design.nlayers, design.dir, design.layer_capacity,
                              design.len_cost, design.via_cost, design.ovf_weight, design.logistic_slope,
                              design.slack_clamp, ecap)
        self.h = fgr_grid_create(self.desc, device, stream)
        torch.cuda.synchronize(self.dev)
        self.hybrid = hybrid
        if hybrid is not None:
            fgr_set_pattern(self.h, hybrid[0], hybrid[1])
        if dp_policy is not None:   # (policy, flow_max)
            fgr_set_dp_policy(self.h, dp_policy[0], dp_policy[1])
        self._ecap = ecap
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(self.dev)
        self.t_off, self.t_x, self.t_y = t(design.node_offset), t(design.x), t(design.y)
        self.t_plo, self.t_phi, self.t_par = t(design.pin_lo), t(design.pin_hi), t(design.parent)
        self.nets = make_nets(design.num_nets, design.num_nodes, self.t_off, self.t_x, self.t_y, self.t_plo,
                              self.t_phi, self.t_par)
        N, M = design.num_nets, design.num_nodes
        i32 = torch.int32
        self.batch_of_net = torch.empty(max(N, 1), dtype=i32, device=self.dev)
        self.order = torch.empty(max(N, 1), dtype=i32, device=self.dev)
        self.batch_offset = torch.empty(N + 1, dtype=i32, device=self.dev)
        self.seg = torch.empty(max(M, 1), dtype=i32, device=self.dev)
        self.zmid = torch.full((max(M, 1),), -1, dtype=i32, device=self.dev)
        self.cost = torch.empty(max(N, 1), dtype=i32, device=self.dev)
        self.num_batches = 0

    def close(self):
        if self.h:
            fgr_grid_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def reset_demand(self, demand=None, stream=None):
        fgr_grid_set_demand(self.h, demand, stream)

    def plan(self, stream=None) -> int:
        self.num_batches = fgr_plan(self.h, self.nets, self.batch_of_net, self.order, self.batch_offset, stream)
        return self.num_batches

    def route_all(self, stream=None):
        if self.hybrid is None:
            fgr_route_all(self.h, self.nets, self.order, self.batch_offset, self.num_batches, self.seg, self.cost,
                          stream)
        else:
            fgr_route_all_ex(self.h, self.nets, self.order, self.batch_offset, self.num_batches, self.seg, self.zmid,
                             self.cost, stream)

    def route_batch(self, net_ids, stream=None):
        if self.hybrid is None:
            fgr_route_batch(self.h, self.nets, net_ids, int(net_ids.numel()), self.seg, self.cost, stream)
        else:
            fgr_route_batch_ex(self.h, self.nets, net_ids, int(net_ids.numel()), self.seg, self.zmid, self.cost,
                               stream)

    def demand(self, stream=None):
        out = self.torch.empty((self.d.nlayers, self.d.ny, self.d.nx), dtype=self.torch.int32, device=self.dev)
        fgr_grid_get_demand(self.h, out, stream)
        return out

    def run(self, stream=None):
        """Whole stage from zero demand: set_demand(NULL) -> plan -> route_all."""
        self.reset_demand(None, stream)
        self.plan(stream)
        self.route_all(stream)

    def results(self):
        """(batch_of_net, num_batches, seg uint32, cost uint32, demand) as host numpy arrays."""
        self.torch.cuda.synchronize(self.dev)
        N, M = self.d.num_nets, self.d.num_nodes
        return (self.batch_of_net[:N].cpu().numpy(), self.num_batches,
                self.seg[:M].cpu().numpy().view(np.uint32), self.cost[:N].cpu().numpy().view(np.uint32),
                self.demand().cpu().numpy())

    def overflow(self, stream=None):
        """Rip-up set of the last route call -> (violating uint8[N], rip_ids int32[R], totals) on the host."""
        torch = self.torch
        N = self.d.num_nets
        viol = torch.empty(max(N, 1), dtype=torch.uint8, device=self.dev)
        rip = torch.empty(max(N, 1), dtype=torch.int32, device=self.dev)
        nr, tot = fgr_overflow(self.h, self.nets, self.seg, self.zmid if self.hybrid is not None else None, viol, rip,
                               stream)
        return viol[:N].cpu().numpy(), rip[:nr].cpu().numpy(), tot

    def task_graph(self, tasks, stream=None):
        """Ordered task graph of net ids `tasks` (host array) -> (order, is_root, succ_offset, succ) on the host."""
        torch = self.torch
        t = torch.from_numpy(np.ascontiguousarray(tasks, np.int32)).to(self.dev)
        R = int(t.numel())
        order = torch.empty(max(R, 1), dtype=torch.int32, device=self.dev)
        root = torch.empty(max(R, 1), dtype=torch.uint8, device=self.dev)
        off = torch.empty(R + 1, dtype=torch.int32, device=self.dev)
        cap = 1 << 16
        while True:
            succ = torch.empty(cap, dtype=torch.int32, device=self.dev)
            try:
                ne = fgr_task_graph(self.h, self.nets, t, R, order, root, off, succ, cap, stream)
                break
            except FgrError as e:
                if e.status != FGR_ERR_RANGE:
                    raise
                cap *= 4
        return (order[:R].cpu().numpy(), root[:R].cpu().numpy(), off.cpu().numpy(), succ[:ne].cpu().numpy())

    def zmids(self):
        """zmid int32[M] (mid | lb << 16 of Z routes, -1 elsewhere) of the last hybrid route call."""
        self.torch.cuda.synchronize(self.dev)
        return self.zmid[:self.d.num_nodes].cpu().numpy()
