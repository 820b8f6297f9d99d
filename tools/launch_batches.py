"""Per-batch critical path from an ncu launch list (serialised kernel times): refresh + max(DP kernels of the batch)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = next(r for r in rows if r and r[0] == "ID")
ks = []
for r in rows:
    if len(r) == len(hdr) and r[0] != "ID":
        d = dict(zip(hdr, r))
        ks.append((d["Kernel Name"].split("(")[0].replace("void ", "").replace("<unnamed>::", ""), float(d["Metric Value"]) / 1000))
# last step only: from the last k_preprocess on
start = max(i for i, k in enumerate(ks) if k[0].startswith("k_preprocess"))
ks = ks[start:]
batches, cur = [], None
plan = 0.0
for name, us in ks:
    if name.startswith("k_refresh"):
        cur = {"refresh": us, "dp": {}}
        batches.append(cur)
    elif cur is None:
        plan += us
    elif name.startswith("k_dp") or name.startswith("k_hyb"):
        cur["dp"][name] = cur["dp"].get(name, 0) + us
tot_crit = sum(b["refresh"] + max(b["dp"].values() or [0]) for b in batches)
print(f"plan kernels {plan:.0f} us, batches {len(batches)}, sum(refresh + max dp) = {tot_crit:.0f} us")
acc = 0
for i, b in enumerate(batches):
    crit = b["refresh"] + max(b["dp"].values() or [0])
    acc += crit
    if i < 12 or i % 8 == 0:
        print(f"b={i:3d} crit {crit:7.1f}  acc {acc:8.0f}  refresh {b['refresh']:6.1f}  " + "  ".join(f"{k[5:]}={v:.0f}" for k, v in sorted(b["dp"].items())))
