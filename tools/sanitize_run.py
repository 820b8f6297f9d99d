"""Small end-to-end runs for compute-sanitizer (memcheck / racecheck / synccheck), every DP kernel:
k_dp_two / k_dp_walk (tiny), k_dp_flow with its root-path walker and k_dp_large (bignets, chains),
k_dp_hld (huge: nets above the shared-memory limit; and every large net under FGR_DP_HLD),
hybrid L+Z (k_hyb_tm), the emulated exchange path, fgr_overflow / fgr_task_graph.
Usage: python tools/sanitize_run.py [small|all]"""
import sys
sys.path.insert(0, ".")
import numpy as np
import gen
from oracle import Oracle
from paper_conf_date_liulzclly22_b200 import Router
from paper_conf_date_liulzclly22_b200 import fastgr as F

which = sys.argv[1] if len(sys.argv) > 1 else "all"
designs = [("tiny", gen.make_config("tiny"), None, None, 0),
           ("bignets", gen.generate(nx=60, ny=50, nlayers=9, num_nets=40, seed=77, caps=gen.CAP9, pin_dist=1, kmin=30,
                                    kmax=120, hpwl_base=12.0, hpwl_sigma=0.5, name="bignets"), None, None, 0),
           ("bignets-hld", gen.generate(nx=60, ny=50, nlayers=9, num_nets=40, seed=77, caps=gen.CAP9, pin_dist=1, kmin=30,
                                        kmax=120, hpwl_base=12.0, hpwl_sigma=0.5, name="bignets"), None,
            (F.FGR_DP_HLD, 64), 0),
           ("t1-hybrid-exchange", gen.make_config("t1", num_nets=400), (10, 500), None, 2)]
if which == "all":
    designs += [("chains", gen.generate(nx=160, ny=150, nlayers=9, num_nets=12, seed=91, caps=gen.CAP9, pin_dist=1,
                                        kmin=300, kmax=900, hpwl_base=60.0, hpwl_sigma=0.3, name="chains"),
                 None, (F.FGR_DP_AUTO, 65535), 0),
                ("huge", gen.generate(nx=300, ny=300, nlayers=9, num_nets=3, seed=5, caps=gen.CAP9, pin_dist=1,
                                      kmin=1400, kmax=3000, hpwl_base=120.0, hpwl_sigma=0.2, name="huge"), None, None, 0)]
bad = 0
for name, d, hyb, pol, emu in designs:
    r = Router(d, hybrid=hyb, dp_policy=pol)
    if emu:
        F.fgr_set_exchange(r.h, 0, emu)
    r.run()
    b, nb, seg, cost, dem = r.results()
    o = Oracle(d)
    ob, onb = o.plan()
    if hyb:
        oseg, ocost, odem = o.route(ob, onb, hybrid=hyb)
    else:
        oseg, ocost, odem = o.route(ob, onb)
    ok = nb == onb and np.array_equal(b, ob) and np.array_equal(seg, oseg) and np.array_equal(dem, odem)
    viol, rip, tot = r.overflow()
    if len(rip):
        r.task_graph(rip)
    print(name, "batches", nb, "parity", ok, "rip", len(rip), flush=True)
    bad += not ok
    r.close()
sys.exit(1 if bad else 0)
