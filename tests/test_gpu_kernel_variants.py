"""GPU parity of every large-net DP kernel selection (fgr_set_dp_policy, include/fastgr.h;
DESIGN.md §5): the tree-dataflow kernel (k_dp_flow) up to flow_max nodes, the heavy-path
kernel (k_dp_large) up to its shared-memory limit, the heavy-path contraction kernel
(k_dp_hld) above it or for every net.  Each selection is checked element by element against
the oracle through fgr_route_all (with the once-per-stage tree analyses) and fgr_route_batch
(without them).

The "chains" design has large nets with long root paths (>= 64 nodes, the flow kernel's
root-path walker); "huge" has nets of 1.5k-4.4k nodes, above the shared-memory kernels' limit.
"""
import sys

import numpy as np
import pytest

import gen
from oracle import Oracle
from paper_conf_date_liulzclly22_b200 import fastgr as F

pytestmark = pytest.mark.gpu

DESIGNS = {
    "t5": lambda: gen.make_config("t5", num_nets=20000),
    "bignets": lambda: gen.generate(nx=120, ny=110, nlayers=9, num_nets=400, seed=77, caps=gen.CAP9, pin_dist=1,
                                    kmin=30, kmax=400, hpwl_base=20.0, hpwl_sigma=0.5, name="bignets"),
    "chains": lambda: gen.generate(nx=160, ny=150, nlayers=9, num_nets=120, seed=91, caps=gen.CAP9, pin_dist=1,
                                   kmin=300, kmax=900, hpwl_base=60.0, hpwl_sigma=0.3, name="chains"),
    "huge": lambda: gen.generate(nx=300, ny=300, nlayers=9, num_nets=12, seed=5, caps=gen.CAP9, pin_dist=1,
                                 kmin=1400, kmax=5000, hpwl_base=160.0, hpwl_sigma=0.2, name="huge"),
}

POLICIES = {
    "auto": (F.FGR_DP_AUTO, 64),
    "flow_all": (F.FGR_DP_AUTO, 65535),
    "flow_40": (F.FGR_DP_AUTO, 40),
    "heavy": (F.FGR_DP_HEAVY, 64),
    "hld": (F.FGR_DP_HLD, 64),
}

_cache = {}


def _oracle(name):
    if name not in _cache:
        d = DESIGNS[name]()
        o = Oracle(d)
        ob, onb = o.plan()
        _cache[name] = (d, ob, onb) + tuple(o.route(ob, onb))
    return _cache[name]


def first_diff(a, b):
    idx = np.nonzero(a != b)[0]
    return None if len(idx) == 0 else (int(idx[0]), a[idx[0]], b[idx[0]], len(idx))


@pytest.mark.parametrize("policy", sorted(POLICIES))
@pytest.mark.parametrize("design", sorted(DESIGNS))
def test_kernel_selection_bit_exact(policy, design):
    import torch
    d, ob, onb, oseg, ocost, odem = _oracle(design)
    r = F.Router(d, device=0, dp_policy=POLICIES[policy])
    r.reset_demand(None)
    nb = r.plan()
    r.route_all()
    b, nb, seg, cost, dem = r.results()
    assert nb == onb
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(cost, ocost), first_diff(cost, ocost)
    assert np.array_equal(dem, odem)
    # fgr_route_batch: no once-per-stage analyses (the kernels build their tables themselves)
    r.reset_demand(None)
    r.seg.fill_(-1)
    r.cost.zero_()
    for bb in range(onb):
        r.route_batch(torch.from_numpy(np.nonzero(ob == bb)[0].astype(np.int32)).cuda())
    torch.cuda.synchronize()
    seg = r.seg.cpu().numpy().view(np.uint32)
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(r.cost.cpu().numpy().view(np.uint32), ocost)
    assert np.array_equal(r.demand().cpu().numpy(), odem)
    r.close()


def test_designs_reach_the_intended_kernels():
    """chains: root paths >= 64 nodes (flow kernel's walker); huge: nets above the 1.3k-node shared-memory limit."""
    d = DESIGNS["chains"]()
    sizes = d.net_sizes()
    deepest = 0
    for n in np.nonzero(sizes > 128)[0][:20]:
        a = d.node_offset[n]
        par = d.parent[a:a + sizes[n]]
        depth = np.zeros(sizes[n], np.int64)
        for i in range(1, sizes[n]):
            depth[i] = depth[par[i]] + 1
        deepest = max(deepest, int(depth.max()))
    assert deepest >= 64, deepest
    assert (DESIGNS["huge"]().net_sizes() > 1400).sum() >= 10


def test_dp_policy_validation():
    d = gen.make_config("tiny", num_nets=5)
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    r = F.Router(d, device=0)
    with pytest.raises(F.FgrError):
        F.fgr_set_dp_policy(r.h, 7, 64)
    with pytest.raises(F.FgrError):
        F.fgr_set_dp_policy(r.h, F.FGR_DP_AUTO, 8)
    r.close()
