"""Route one design (default: chains) twice through route_all; used under ncu to capture the large-net DP
launches.  Usage: python tools/prof_hld.py [chains|t9] [auto|heavy|hld]"""
import sys
sys.path.insert(0, ".")
import torch
import gen
from paper_conf_date_liulzclly22_b200 import Router
from paper_conf_date_liulzclly22_b200.fastgr import FGR_DP_AUTO, FGR_DP_HEAVY, FGR_DP_HLD

name = sys.argv[1] if len(sys.argv) > 1 else "chains"
pol = {"auto": FGR_DP_AUTO, "heavy": FGR_DP_HEAVY, "hld": FGR_DP_HLD}[sys.argv[2] if len(sys.argv) > 2 else "auto"]
designs = {
    "chains": lambda: gen.generate(nx=160, ny=150, nlayers=9, num_nets=120, seed=91, caps=gen.CAP9, pin_dist=1,
                                   kmin=300, kmax=900, hpwl_base=60.0, hpwl_sigma=0.3, name="chains"),
    "t9": lambda: gen.make_config("t9"),
}
d = designs[name]()
r = Router(d, device=0, dp_policy=(pol, 64))
for it in range(2):
    r.reset_demand(None)
    r.plan()
    r.route_all()
    torch.cuda.synchronize()
print("done")
