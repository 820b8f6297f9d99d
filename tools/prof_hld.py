"""Route one design (default: chains) twice through route_all; used under ncu to capture k_dp_hld launches."""
import sys
sys.path.insert(0, ".")
import torch
import gen
from tests.test_gpu_parity import _router

name = sys.argv[1] if len(sys.argv) > 1 else "chains"
designs = {
    "chains": lambda: gen.generate(nx=160, ny=150, nlayers=9, num_nets=120, seed=91, caps=gen.CAP9, pin_dist=1,
                                   kmin=300, kmax=900, hpwl_base=60.0, hpwl_sigma=0.3, name="chains"),
    "t9": lambda: gen.make_config("t9"),
}
d = designs[name]()
r = _router(d)
for it in range(2):
    r.reset_demand(None)
    r.plan()
    r.route_all()
    torch.cuda.synchronize()
print("done")
