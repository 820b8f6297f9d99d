"""GPU parity of the multi-GPU exchange path and of the host-buffer end-to-end call.

* fgr_route_all's exchange path (include/fastgr.h) — split each
  batch by tree edges (fgr_split_batch), route every rank's chunk into the route
  records, commit every net of the batch from the records — run on one GPU with
  k emulated ranks (fgr_set_exchange's emulate_world): all ranks' chunks land in one
  record buffer, which is then exactly what the NCCL SUM all-reduce produces.  This
  executes the split arithmetic, the record offsets of ranks > 0 and the partial
  large/small launches that a world-1 communicator never reaches.  Batches below
  split_min take the whole-batch path (routed and committed by the DP kernels).
* fgr_run_host / fgr_run_host_ex (pinned host nets in -> plan -> route -> seg, zmid,
  cost out), the call behind bench.py's e2e number.
Every output is compared with the oracle element by element.
"""
import numpy as np
import pytest

import gen
from oracle import Oracle
from paper_conf_date_liulzclly22_b200 import fastgr as F

pytestmark = pytest.mark.gpu

DESIGNS = {
    "tiny": lambda: gen.make_config("tiny"),
    "t5": lambda: gen.make_config("t5"),
    "bignets": lambda: gen.generate(nx=120, ny=110, nlayers=9, num_nets=400, seed=77, caps=gen.CAP9, pin_dist=1,
                                    kmin=30, kmax=400, hpwl_base=20.0, hpwl_sigma=0.5, name="bignets"),
    "huge": lambda: gen.generate(nx=300, ny=300, nlayers=9, num_nets=12, seed=5, caps=gen.CAP9, pin_dist=1,
                                 kmin=1400, kmax=5000, hpwl_base=160.0, hpwl_sigma=0.2, name="huge"),
}
HYB = (10, 500)   # hybrid window selecting ~1% of the synthetic edges (R23)
_cache = {}


def _oracle(name, hybrid=None):
    key = (name, hybrid)
    if key not in _cache:
        d = DESIGNS[name]()
        o = Oracle(d)
        ob, onb = o.plan()
        if hybrid is None:
            res = o.route(ob, onb) + (None,)
        else:
            res = o.route(ob, onb, hybrid=hybrid, with_zmid=True)
        _cache[key] = (d, onb) + tuple(res)
    return _cache[key]


def first_diff(a, b):
    idx = np.nonzero(a != b)[0]
    return None if len(idx) == 0 else (int(idx[0]), a[idx[0]], b[idx[0]], len(idx))


def _check(r, onb, oseg, ocost, odem, ozmid=None):
    b, nb, seg, cost, dem = r.results()
    assert nb == onb
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(cost, ocost), first_diff(cost, ocost)
    assert np.array_equal(dem, odem), first_diff(dem.ravel(), odem.ravel())
    if ozmid is not None:
        z = r.zmids()
        assert np.array_equal(z, ozmid), first_diff(z, ozmid)


@pytest.mark.parametrize("world", [2, 3, 8])
@pytest.mark.parametrize("design", ["tiny", "t5", "bignets", "huge"])
def test_emulated_ranks_bit_exact(design, world):
    d, onb, oseg, ocost, odem, _ = _oracle(design)
    r = F.Router(d, device=0)
    F.fgr_set_exchange(r.h, 0, world)   # split every batch
    r.run()
    _check(r, onb, oseg, ocost, odem)
    st = F.fgr_get_stats(r.h)
    assert st["exchanged_batches"] == onb
    r.close()


@pytest.mark.parametrize("world", [2, 3])
def test_emulated_ranks_hybrid_bit_exact(world):
    d, onb, oseg, ocost, odem, ozmid = _oracle("t5", HYB)
    r = F.Router(d, device=0, hybrid=HYB)
    F.fgr_set_exchange(r.h, 0, world)
    r.run()
    _check(r, onb, oseg, ocost, odem, ozmid)
    r.close()


def test_emulated_ranks_whole_batch_path():
    """split_min above every batch: all batches routed whole (no exchange), still bit-exact;
    an intermediate split_min mixes both paths."""
    d, onb, oseg, ocost, odem, _ = _oracle("t5")
    for split_min, expect_all_whole in ((1 << 30, True), (500, False)):
        r = F.Router(d, device=0)
        F.fgr_set_exchange(r.h, split_min, 2)
        r.run()
        _check(r, onb, oseg, ocost, odem)
        st = F.fgr_get_stats(r.h)
        if expect_all_whole:
            assert st["exchanged_batches"] == 0
        else:
            assert 0 < st["exchanged_batches"] < onb
        r.close()


@pytest.mark.parametrize("cfg,hybrid", [("t1", None), ("t1", HYB), ("t9", None)])
def test_run_host_bit_exact(cfg, hybrid):
    """fgr_run_host(_ex): host nets in (pinned), seg / zmid / cost / num_batches out."""
    import torch
    d = gen.make_config(cfg)
    o = Oracle(d)
    ob, onb = o.plan()
    if hybrid is None:
        oseg, ocost, odem = o.route(ob, onb)
        ozmid = None
    else:
        oseg, ocost, odem, ozmid = o.route(ob, onb, hybrid=hybrid, with_zmid=True)
    r = F.Router(d, device=0, hybrid=hybrid)
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
    args = [pin(d.node_offset), pin(d.x), pin(d.y), pin(d.pin_lo), pin(d.pin_hi), pin(d.parent)]
    seg = torch.empty(d.num_nodes, dtype=torch.int32).pin_memory()
    cost = torch.empty(d.num_nets, dtype=torch.int32).pin_memory()
    if hybrid is None:
        nb = F.fgr_run_host(r.h, *args, seg_out=seg, net_cost=cost)
    else:
        zmid = torch.full((d.num_nodes,), 12345, dtype=torch.int32).pin_memory()
        nb = F.fgr_run_host_ex(r.h, *args, seg_out=seg, zmid_out=zmid, net_cost=cost)
        z = zmid.numpy()
        assert np.array_equal(z, ozmid), first_diff(z, ozmid)
    assert nb == onb
    s = seg.numpy().view(np.uint32)
    c = cost.numpy().view(np.uint32)
    assert np.array_equal(s, oseg), first_diff(s, oseg)
    assert np.array_equal(c, ocost), first_diff(c, ocost)
    dem = r.demand().cpu().numpy()
    assert np.array_equal(dem, odem)
    r.close()
