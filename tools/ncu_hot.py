"""Summarise an ncu report's SASS page: top instructions by stall samples + stall totals."""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
lines = out.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"Address"'))
rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
tot = {}
for r in rows:
    for k, v in r.items():
        if k.startswith("stall_") and "Not Issued" not in k:
            try:
                tot[k] = tot.get(k, 0) + int(v)
            except ValueError:
                pass
S = sum(tot.values())
print("stall totals:", ", ".join(f"{k[6:]}={v/S:.1%}" for k, v in sorted(tot.items(), key=lambda x: -x[1])[:8]))
order = list(range(len(rows)))
order.sort(key=lambda i: -int(rows[i]["Warp Stall Sampling (All Samples)"] or 0))
for i in order[:top]:
    r = rows[i]
    st = sorted(((k[6:], int(v)) for k, v in r.items() if k.startswith("stall_") and "Not Issued" not in k and v.isdigit() and int(v) > 0), key=lambda x: -x[1])[:3]
    print(f'{int(r["Warp Stall Sampling (All Samples)"]):6d} #{i:5d} {r["Source"].strip()[:58]:58s} {st}')

if len(sys.argv) > 3:
    cuts = [int(c) for c in sys.argv[3].split(",")]
    buckets = [0] * (len(cuts) + 1)
    for i, r in enumerate(rows):
        k = sum(1 for c in cuts if i >= c)
        buckets[k] += int(r["Warp Stall Sampling (All Samples)"] or 0)
    T = sum(buckets)
    print("range shares:", [f"{b/T:.1%}" for b in buckets])
