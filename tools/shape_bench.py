"""Route single synthetic large nets of fixed shapes (path, comb) to measure the tree kernel's per-step latency
(use with FGR_LIB_PATH=build_t/libfastgr_tt.so for the per-phase prints).  Usage: python tools/shape_bench.py [path|comb] [m]"""
import sys
import numpy as np
sys.path.insert(0, ".")
import torch
import gen
from paper_conf_date_liulzclly22_b200 import Router

shape = sys.argv[1] if len(sys.argv) > 1 else "path"
m = int(sys.argv[2]) if len(sys.argv) > 2 else 900
n = 1000
x = np.zeros(m, np.int16); y = np.zeros(m, np.int16); par = np.full(m, -1, np.int32)
if shape == "path":   # zig-zag staircase: every edge a bent L, every node one child
    for i in range(m):
        x[i] = 10 + (i + 1) // 2; y[i] = 10 + i // 2; par[i] = i - 1
else:                 # comb: a staircase spine with a one-node tooth on every spine node
    k = m // 2
    for i in range(k):
        x[i] = 10 + (i + 1) // 2; y[i] = 10 + i // 2; par[i] = i - 1
    for j in range(m - k):
        x[k + j] = x[j] + 3; y[k + j] = y[j] + 5 if y[j] + 5 < n else y[j] - 5; par[k + j] = j
par[0] = -1
d = gen.Design(nx=n, ny=n, nlayers=9, dir=np.array([l % 2 for l in range(9)], np.uint8),
               layer_capacity=np.array(gen.CAP9, np.int32), edge_capacity=None,
               node_offset=np.array([0, m], np.int32), x=x, y=y, pin_lo=np.full(m, -1, np.int8),
               pin_hi=np.full(m, -1, np.int8), parent=par, name=shape)
r = Router(d, device=0)
for it in range(3):
    r.reset_demand(None)
    r.plan()
    st = torch.cuda.Event(enable_timing=True); en = torch.cuda.Event(enable_timing=True)
    st.record(); r.route_all(); en.record(); torch.cuda.synchronize()
    print(shape, m, "route_all ms", round(st.elapsed_time(en), 3), flush=True)
