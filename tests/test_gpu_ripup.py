"""GPU parity of the rip-up extraction and the ordered task graph.

fgr_overflow (R26) and fgr_task_graph (§III-B
L414-466; R27) through the C ABI vs. oracle.overflow / oracle.task_graph:
violating flags, rip-up ids, overflow totals, task order, root batch and the
successor CSR are bit-exact.
"""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.helpers import design_from_json, load_golden

pytestmark = pytest.mark.gpu


def run_and_check(d, hybrid=None, tg=True):
    from paper_conf_date_liulzclly22_b200 import Router
    r = Router(d, device=0, hybrid=hybrid)
    r.run()
    b, nb, seg, cost, dem = r.results()
    viol, rip, tot = r.overflow()
    o = Oracle(d)
    ob, onb = o.plan()
    oseg, ocost, odem, oz = o.route(ob, onb, hybrid=hybrid, with_zmid=True)
    assert np.array_equal(seg, oseg) and np.array_equal(dem, odem)
    oviol, otot = o.overflow(oseg, odem, oz)
    assert tot == otot, (tot, otot)
    assert np.array_equal(viol, oviol)
    assert np.array_equal(rip, np.nonzero(oviol)[0].astype(np.int32))
    if tg:
        order, root, off, succ = r.task_graph(rip)
        oo, oroot, ooff, osucc = o.task_graph(rip)
        assert np.array_equal(order, oo) and np.array_equal(root, oroot)
        assert np.array_equal(off, ooff) and np.array_equal(succ, osucc)
    r.close()
    return int(viol.sum())


def test_ov1_and_tg1_hand_worked():
    from paper_conf_date_liulzclly22_b200 import Router
    j = load_golden("OV1.json")
    d = design_from_json(j)
    r = Router(d, device=0)
    r.run()
    viol, rip, tot = r.overflow()
    assert list(viol) == j["expect"]["violating"] and list(tot) == j["expect"]["totals"]
    assert list(rip) == [0, 1]
    r.close()
    j = load_golden("TG1.json")
    d = design_from_json(j)
    r = Router(d, device=0)
    order, root, off, succ = r.task_graph(np.arange(d.num_nets))
    e = j["expect"]
    assert list(order) == e["order"] and list(root) == e["is_root"]
    assert list(off) == e["succ_offset"] and list(succ) == e["succ"]
    r.close()


@pytest.mark.parametrize("seed,hybrid", [(0, None), (1, None), (2, (3, 40)), (3, (2, 80))])
def test_random_congested(seed, hybrid):
    L = [4, 5, 9, 6][seed]
    d = gen.random_small(seed=1880 + seed, nx=60 + 10 * seed, ny=50, nlayers=L, num_nets=900, kmax=10,
                         literal_frac=0.3, caps=[1] * L)
    assert run_and_check(d, hybrid) > 20


def test_t1_edge_capacity_override():
    d = gen.make_config("t1")
    rng = np.random.default_rng(7)
    d.edge_capacity = rng.integers(0, 3, size=(d.nlayers, d.ny, d.nx)).astype(np.uint8)
    assert run_and_check(d) > 50


def test_no_overflow_empty_rip_set():
    d = gen.make_config("t5")
    assert run_and_check(d) == 0


def test_t9_full_size_capacity3():
    """Headline config with capacity 3 on layers 1-8: ~10.7k violating nets, ~411k task-graph edges."""
    d = gen.make_config("t9")
    d.layer_capacity = np.array([1, 3, 3, 3, 3, 3, 3, 3, 3], np.int32)
    assert run_and_check(d) > 5000
