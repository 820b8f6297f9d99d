"""One warm step of the stage on a config (for ncu / compute-sanitizer runs)."""
import sys
sys.path.insert(0, ".")
import torch
import gen
from paper_conf_date_liulzclly22_b200 import Router

cfg = sys.argv[1] if len(sys.argv) > 1 else "t9"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
d = gen.make_config(cfg)
r = Router(d)
for _ in range(steps):
    r.run()
torch.cuda.synchronize()
print("batches", r.num_batches)
