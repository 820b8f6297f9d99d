"""Debug helper: find the first net whose GPU route differs from the oracle's and print it."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import gen
from oracle import Oracle
from paper_conf_date_liulzclly22_b200 import Router

cfg = sys.argv[1] if len(sys.argv) > 1 else "tiny"
d = gen.make_config(cfg)
o = Oracle(d)
shown = 0
for n in range(d.num_nets):
    if d.node_offset[n + 1] - d.node_offset[n] < 2:
        continue
    s = d.subset([n])
    r = Router(s)
    r.run()
    b, nb, seg, cost, dem = r.results()
    os_ = Oracle(s)
    ob, onb = os_.plan()
    oseg, ocost, odem = os_.route(ob, onb)
    if not (np.array_equal(seg, oseg) and np.array_equal(cost, ocost) and np.array_equal(dem, odem)):
        print("net", n, "m", s.num_nodes)
        print(" x", s.x, "\n y", s.y, "\n plo", s.pin_lo, "\n phi", s.pin_hi, "\n par", s.parent)
        print(" gpu seg", [hex(v) for v in seg], "cost", cost)
        print(" orc seg", [hex(v) for v in oseg], "cost", ocost)
        print(" dem equal", np.array_equal(dem, odem))
        shown += 1
        if shown > 3:
            break
    r.close()
print("done")
