"""Per-batch device time of route_batch (refresh + DP + commit) vs batch size."""
import sys
sys.path.insert(0, ".")
import numpy as np
import torch
import gen
from paper_conf_date_liulzclly22_b200 import Router
from paper_conf_date_liulzclly22_b200 import fastgr as F

cfg = sys.argv[1] if len(sys.argv) > 1 else "t9"
d = gen.make_config(cfg)
r = Router(d)
r.run()  # warm
r.reset_demand(None)
nb = r.plan()
boff = r.batch_offset[:nb + 1].cpu().numpy()
sizes = d.net_sizes()
order = r.order.cpu().numpy()
F.fgr_profile_enable(r.h, True)
rows = []
for b in range(nb):
    ids = r.order[boff[b]:boff[b + 1]]
    r.route_batch(ids)
    prof = F.fgr_profile_read(r.h)
    ms = order[boff[b]:boff[b + 1]]
    rows.append((b, boff[b + 1] - boff[b], int((sizes[ms] > 32).sum()), int(sizes[ms].max()),
                 prof["refresh"][0] * 1000, prof["dp_small"][0] * 1000, prof["dp_large"][0] * 1000))
F.fgr_profile_enable(r.h, False)
tot = np.array([x[4:] for x in rows]).sum(0)
print("totals us: refresh %.0f small %.0f large %.0f" % tuple(tot))
for x in rows:
    print("b=%3d nets=%7d large=%4d maxm=%5d | refresh %7.1f us  small %7.1f us  large %7.1f us" % x)
