"""Summarise a round's ncu captures (gpurun_out/<tag>_*) into profiles/<tag>_summary.md and
profiles/<tag>_traffic.json (per-launch DRAM bytes per kernel class, read by bench.py)."""
import csv, io, json, os, re, subprocess, sys
from collections import defaultdict

tag = sys.argv[1]
src = sys.argv[2] if len(sys.argv) > 2 else "gpurun_out"
out_md = [f"# ncu summary — {tag}\n"]

def short(name):
    m = re.search(r"(k_\w+?)(?:ILi(\d+)|I|\(|<|$)", name)
    return m.group(1) if m else name[:40]

# 1. launch list
p = f"{src}/{tag}_launches.csv"
if os.path.exists(p):
    rows = [r for r in csv.reader(l for l in open(p) if l.startswith('"'))]
    h = rows[0]; idx = {k: i for i, k in enumerate(h)}
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        if r[idx["Metric Name"]] != "gpu__time_duration.sum":
            continue
        k = short(r[idx["Kernel Name"]])
        agg[k][0] += 1
        agg[k][1] += float(r[idx["Metric Value"]].replace(",", "")) / 1000.0
    tot = sum(v[1] for v in agg.values())
    out_md.append("## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold-cache, serialised)\n")
    out_md.append("Command: `python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e` (2 steps + setup).\n")
    out_md.append("| kernel | launches | total us | share |\n|---|---|---|---|")
    for k, (n, us) in sorted(agg.items(), key=lambda x: -x[1][1]):
        out_md.append(f"| {k} | {n} | {us:.0f} | {us/tot:.1%} |")
    out_md.append("")

# 2. full captures
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__occupancy_limit_registers",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "smsp__inst_executed.sum", "launch__grid_size", "smsp__issue_active.avg.pct_of_peak_sustained_active"]
for f in sorted(os.listdir(src)):
    if not (f.startswith(tag + "_full_") and f.endswith(".ncu-rep")):
        continue
    raw = subprocess.run(["ncu", "-i", f"{src}/{f}", "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(io.StringIO(raw)))
    if len(rr) < 3:
        continue
    h = rr[0]
    out_md.append(f"## {f}\n")
    for row in rr[2:]:
        d = dict(zip(h, row))
        out_md.append(f"- kernel `{short(d.get('Kernel Name',''))}`: " + ", ".join(
            f"{k}={d[k]}" for k in keys if k in d))
    hot = subprocess.run([sys.executable, "tools/ncu_hot.py", f"{src}/{f}", "6"], capture_output=True, text=True).stdout
    out_md.append("\n```\n" + hot.strip() + "\n```\n")

# 3. per-launch traffic
p = f"{src}/{tag}_traffic.csv"
traffic = {}
if os.path.exists(p):
    rows = [r for r in csv.reader(l for l in open(p) if l.startswith('"'))]
    h = rows[0]; idx = {k: i for i, k in enumerate(h)}
    per = defaultdict(lambda: defaultdict(float))
    for r in rows[1:]:
        k = short(r[idx["Kernel Name"]]); lid = r[idx["ID"]]
        v = float(r[idx["Metric Value"]].replace(",", ""))
        unit = r[idx["Metric Unit"]]
        mul = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6}.get(unit, 1)
        per[(k, lid)][r[idx["Metric Name"]]] += v * mul
    agg = defaultdict(lambda: [0, 0.0, 0.0])
    for (k, lid), m in per.items():
        agg[k][0] += 1
        agg[k][1] += m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        agg[k][2] += m.get("gpu__time_duration.sum", 0)
    cls = {"k_dp_tree": "dp_large", "k_dp_large": "dp_large_heavy", "k_dp_walk": "dp_small", "k_dp_two": "dp_two", "k_refresh": "refresh",
           "k_color": "plan_color", "k_dp_flow": "dp_flow"}
    out_md.append("## DRAM traffic per launch over one t9 step (ncu dram__bytes_read.sum + write.sum)\n")
    out_md.append("| kernel | launches | avg bytes/launch | avg us/launch (serialised) |\n|---|---|---|---|")
    for k, (n, b, t) in agg.items():
        out_md.append(f"| {k} | {n} | {b/n:.0f} | {t/n/1000:.1f} |")
        if k in cls:
            traffic[cls[k]] = b / n
    json.dump({"tag": tag, "bytes_per_launch": traffic, "source": p}, open(f"profiles/{tag}_traffic.json", "w"), indent=1)
os.makedirs("profiles", exist_ok=True)
open(f"profiles/{tag}_summary.md", "w").write("\n".join(out_md) + "\n")
print("\n".join(out_md))
