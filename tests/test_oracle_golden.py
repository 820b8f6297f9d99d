"""Oracle vs. hand-worked examples (tests/golden/*.json, each citing its passage)."""
import numpy as np
import pytest

from oracle import Oracle
from tests.helpers import design_from_json, load_golden, seg_fields, recount_demand, PyCost, route_cost


@pytest.mark.parametrize("name", ["W1.json", "W2.json", "W3.json"])
def test_worked_examples(name):
    j = load_golden(name)
    d = design_from_json(j)
    o = Oracle(d)
    b, nb = o.plan()
    seg, cost, dem = o.route(b, nb)
    assert list(cost) == j["expect"]["total"]
    for n, segs in enumerate(j["expect"]["seg"]):
        a = d.node_offset[n]
        for i, s in enumerate(segs):
            if s is None:
                assert seg[a + i] == 0xFFFFFFFF
            else:
                assert seg_fields(seg[a + i]) == s, (name, i)
    if "demand_plus_one" in j["expect"]:
        want = np.zeros_like(dem)
        for l, y, x in j["expect"]["demand_plus_one"]:
            want[l, y, x] += 1
        assert np.array_equal(dem, want)
    # the reported cost equals the independent re-costing of the chosen route
    pc = PyCost(d, np.zeros_like(dem))
    a, e = d.node_offset[0], d.node_offset[1]
    assert route_cost(d, pc, 0, [None] + list(seg[a + 1:e])) == j["expect"]["total"][0]


def test_w1_reroot():
    """Re-rooting W1 at node 1 gives the same optimum (reading R20)."""
    j = load_golden("W1.json")
    j["nets"][0] = {"x": [2, 0], "y": [1, 0], "pin_lo": [0, 0], "pin_hi": [0, 0], "parent": [-1, 0]}
    d = design_from_json(j)
    o = Oracle(d)
    b, nb = o.plan()
    _, cost, _ = o.route(b, nb)
    assert int(cost[0]) == j["expect"]["reroot_total"]


def test_alg1_example():
    j = load_golden("Aex.json")
    d = design_from_json(j)
    b, nb = Oracle(d).plan()
    assert list(b) == j["expect"]["batch"]
    assert nb == j["expect"]["num_batches"]


def test_logistic_table():
    j = load_golden("logistic_table.json")
    W, S = j["W"], j["S"]
    gj = load_golden("W1.json")
    gj["ovf_weight"] = [W, W]
    gj["logistic_slope"] = j["slope"]
    gj["slack_clamp"] = S
    t = Oracle(design_from_json(gj)).cost_table()
    for s, v in j["values"].items():
        assert t[0, int(s) + S] == v, s
    # logistic symmetry T(s) + T(-s) = W
    for s in range(1, S + 1):
        assert t[0, s + S] + t[0, -s + S] == W
    # monotone non-increasing in slack
    assert np.all(np.diff(t[0]) <= 0)
