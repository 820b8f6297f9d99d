"""GPU parity of every DP kernel selection: the environment switches
FGR_FLOW_MAX (largest net of the dataflow kernel), FGR_LARGE_KERNEL=old and
FGR_GROUP_KERNEL=old are read once per process, so each selection runs in its own
subprocess and is checked element by element against the oracle, through fgr_route_all
(with the once-per-stage tree analysis) and fgr_route_batch (without it).

The "chains" design has large nets with long root paths (>= 64 nodes), so under
FGR_FLOW_MAX=100000 the flow kernel's root-path walker (transfer matrices built by the
worker groups, walker-inline fallback, kicks) is exercised.
"""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import gen
from oracle import Oracle
from tests.test_gpu_parity import check_against_oracle, first_diff, _router

designs = {
    "t5": lambda: gen.make_config("t5", num_nets=20000),
    "bignets": lambda: gen.generate(nx=120, ny=110, nlayers=9, num_nets=400, seed=77, caps=gen.CAP9, pin_dist=1,
                                    kmin=30, kmax=400, hpwl_base=20.0, hpwl_sigma=0.5, name="bignets"),
    "chains": lambda: gen.generate(nx=160, ny=150, nlayers=9, num_nets=120, seed=91, caps=gen.CAP9, pin_dist=1,
                                   kmin=300, kmax=900, hpwl_base=60.0, hpwl_sigma=0.3, name="chains"),
}
for name in sys.argv[1].split(","):
    d = designs[name]()
    check_against_oracle(d)
    # fgr_route_batch: no tree analysis (the kernels build their child CSR themselves)
    o = Oracle(d)
    ob, onb = o.plan()
    oseg, ocost, odem = o.route(ob, onb)
    r = _router(d)
    r.reset_demand(None)
    r.seg.fill_(-1)
    r.cost.zero_()
    for b in range(onb):
        r.route_batch(torch.from_numpy(np.nonzero(ob == b)[0].astype(np.int32)).cuda())
    torch.cuda.synchronize()
    seg = r.seg.cpu().numpy().view(np.uint32)
    assert np.array_equal(seg, oseg), (name, first_diff(seg, oseg))
    assert np.array_equal(r.cost.cpu().numpy().view(np.uint32), ocost), name
    assert np.array_equal(r.demand().cpu().numpy(), odem), name
    r.close()
    print("ok", name, int((d.net_sizes() > 32).sum()), "large nets")
"""

VARIANTS = {
    "flow_all": {"FGR_FLOW_MAX": "100000"},
    "flow_40": {"FGR_FLOW_MAX": "40"},
    "flow_128": {"FGR_FLOW_MAX": "128"},    # the previous default cut
    "large_old": {"FGR_LARGE_KERNEL": "old"},
    "group_old": {"FGR_GROUP_KERNEL": "old"},
}


@pytest.mark.parametrize("variant", sorted(VARIANTS))
def test_kernel_selection_bit_exact(variant):
    env = dict(os.environ)
    env.update(VARIANTS[variant])
    designs = "t5,bignets,chains"
    p = subprocess.run([sys.executable, "-c", SCRIPT, designs], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=900)
    assert p.returncode == 0, p.stdout[-3000:] + p.stderr[-3000:]
    assert p.stdout.count("ok ") == 3, p.stdout


def test_chains_design_has_long_root_paths():
    """The chains design must reach the walker (root path >= 64 nodes)."""
    import numpy as np
    sys.path.insert(0, ROOT)
    import gen
    d = gen.generate(nx=160, ny=150, nlayers=9, num_nets=120, seed=91, caps=gen.CAP9, pin_dist=1, kmin=300, kmax=900,
                     hpwl_base=60.0, hpwl_sigma=0.3, name="chains")
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
