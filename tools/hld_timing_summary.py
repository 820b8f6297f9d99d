"""Summarise FGR_HLD_TIMING prints (per-phase clock64 cycles of k_dp_hld, nets > 500 nodes)."""
import json, re, statistics, sys
t = open(sys.argv[1]).read()
rows = [{k: int(v) for k, v in re.findall(r'(\w+)=(\d+)', l)} for l in t.split('\n') if 'HLD m=' in l]
rows.sort(key=lambda r: -r['m'])
for r in rows[:5]:
    print(r)
for k in ["load","gather","p2","p3a","p3b","p4","p5","p6","total"]:
    print(k, int(statistics.mean(r[k] for r in rows)))
