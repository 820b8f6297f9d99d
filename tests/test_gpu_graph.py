"""The CUDA-Graph replay of fgr_route_all's single-GPU batch loop (fgr_set_graph) gives the
oracle's routes and demand on every call: the first call runs the loop directly, the second
captures it, later calls replay it.  A changed plan (another design on the same grid object) or
the graph switched off falls back to the direct loop.  Batches stay sequential (PAPER.md
L504-512); the graph only removes host issue cost."""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.test_gpu_parity import first_diff

pytestmark = pytest.mark.gpu


def _oracle_routes(d, hybrid=None):
    o = Oracle(d)
    ob, onb = o.plan()
    if hybrid is None:
        seg, cost, dem = o.route(ob, onb)
    else:
        seg, cost, dem = o.route(ob, onb, hybrid=hybrid)[:3]
    return seg, cost, dem


def _route(r):
    r.reset_demand(None)
    r.plan()
    r.route_all()
    _, _, seg, cost, dem = r.results()
    return seg, cost, dem


@pytest.mark.parametrize("cfg", ["t1", "t5"])
def test_graph_replay_bit_exact(cfg):
    from paper_conf_date_liulzclly22_b200 import Router
    d = gen.make_config(cfg) if cfg == "t1" else gen.make_config("t5", num_nets=20000)
    oseg, ocost, odem = _oracle_routes(d)
    from paper_conf_date_liulzclly22_b200.fastgr import fgr_get_stats
    r = Router(d, device=0)
    for it in range(4):   # direct, capture, replay, replay
        seg, cost, dem = _route(r)
        from paper_conf_date_liulzclly22_b200.fastgr import lib
        assert fgr_get_stats(r.h)["graph_mode"] == [0, 1, 2, 2][it], lib().fgr_last_error().decode()
        assert np.array_equal(seg, oseg), (it, first_diff(seg, oseg))
        assert np.array_equal(cost, ocost), (it, first_diff(cost, ocost))
        assert np.array_equal(dem, odem), (it, first_diff(dem.ravel(), odem.ravel()))
    r.close()


def test_graph_off_and_hybrid():
    from paper_conf_date_liulzclly22_b200 import Router
    from paper_conf_date_liulzclly22_b200.fastgr import fgr_set_graph
    d = gen.make_config("t1")
    oseg, ocost, odem = _oracle_routes(d, hybrid=(10, 500))
    r = Router(d, device=0, hybrid=(10, 500))
    for it in range(3):
        seg, cost, dem = _route(r)
        assert np.array_equal(seg, oseg) and np.array_equal(cost, ocost) and np.array_equal(dem, odem), it
    fgr_set_graph(r.h, False)
    seg, cost, dem = _route(r)
    assert np.array_equal(seg, oseg) and np.array_equal(cost, ocost) and np.array_equal(dem, odem)
    r.close()
