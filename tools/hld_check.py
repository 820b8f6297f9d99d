"""Quick GPU check of the large-net DP against the oracle (route_all and route_batch) on designs
with many large nets; prints the first difference.  Usage: python tools/hld_check.py bignets,chains,t5"""
import sys, time
import numpy as np
sys.path.insert(0, ".")
import torch
import gen
from oracle import Oracle
from tests.test_gpu_parity import first_diff, _router

designs = {
    "t5": lambda: gen.make_config("t5", num_nets=20000),
    "t1": lambda: gen.make_config("t1"),
    "bignets": lambda: gen.generate(nx=120, ny=110, nlayers=9, num_nets=400, seed=77, caps=gen.CAP9, pin_dist=1,
                                    kmin=30, kmax=400, hpwl_base=20.0, hpwl_sigma=0.5, name="bignets"),
    "chains": lambda: gen.generate(nx=160, ny=150, nlayers=9, num_nets=120, seed=91, caps=gen.CAP9, pin_dist=1,
                                   kmin=300, kmax=900, hpwl_base=60.0, hpwl_sigma=0.3, name="chains"),
    "huge": lambda: gen.generate(nx=300, ny=300, nlayers=9, num_nets=12, seed=5, caps=gen.CAP9, pin_dist=1,
                                 kmin=1400, kmax=5000, hpwl_base=160.0, hpwl_sigma=0.2, name="huge"),
}
bad = 0
for name in sys.argv[1].split(","):
    d = designs[name]()
    o = Oracle(d)
    ob, onb = o.plan()
    t = time.time()
    oseg, ocost, odem = o.route(ob, onb)
    tor = time.time() - t
    r = _router(d)
    r.reset_demand(None)
    nb = r.plan()
    r.route_all()
    b, nb, seg, cost, dem = r.results()
    ok = np.array_equal(seg, oseg) and np.array_equal(cost, ocost) and np.array_equal(dem, odem)
    print(name, "route_all", "OK" if ok else "DIFF", "seg", first_diff(seg, oseg), "cost", first_diff(cost, ocost),
          "dem", first_diff(dem.ravel(), odem.ravel()), "maxm", int(d.net_sizes().max()), "oracle_s", round(tor, 2), flush=True)
    bad += not ok
    if not ok:
        idx = np.nonzero(seg != oseg)[0]
        sz = d.net_sizes()
        nets = np.searchsorted(d.node_offset, idx, side="right") - 1
        u = np.unique(nets)
        print("  nets with seg diffs:", len(u), "sizes", sz[u][:10], "cost diffs", int((cost != ocost).sum()))
    r.reset_demand(None)
    r.seg.fill_(-1)
    r.cost.zero_()
    for bb in range(onb):
        r.route_batch(torch.from_numpy(np.nonzero(ob == bb)[0].astype(np.int32)).cuda())
    torch.cuda.synchronize()
    seg = r.seg.cpu().numpy().view(np.uint32)
    ok = np.array_equal(seg, oseg) and np.array_equal(r.cost.cpu().numpy().view(np.uint32), ocost)
    print(name, "route_batch", "OK" if ok else "DIFF", first_diff(seg, oseg), flush=True)
    bad += not ok
    r.close()
sys.exit(1 if bad else 0)
