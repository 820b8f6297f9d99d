"""Small end-to-end run for compute-sanitizer (memcheck / racecheck / synccheck)."""
import sys
sys.path.insert(0, ".")
import numpy as np
import gen
from oracle import Oracle
from paper_conf_date_liulzclly22_b200 import Router

designs = [gen.make_config("tiny"),
           gen.generate(nx=60, ny=50, nlayers=9, num_nets=40, seed=77, caps=gen.CAP9, pin_dist=1, kmin=30,
                        kmax=120, hpwl_base=12.0, hpwl_sigma=0.5, name="bignets")]
for d in designs:
    r = Router(d)
    r.run()
    b, nb, seg, cost, dem = r.results()
    ob, onb = Oracle(d).plan()
    oseg, ocost, odem = Oracle(d).route(ob, onb)
    ok = nb == onb and np.array_equal(b, ob) and np.array_equal(seg, oseg) and np.array_equal(dem, odem)
    print(d.name, "batches", nb, "parity", ok)
    r.close()
