"""Instructions executed (and stall samples) per CUDA source line of an ncu report (needs -lineinfo)."""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(r for r in rows if r and r[0] == "Line No")
ie = hdr.index("Instructions Executed")
ws = hdr.index("Warp Stall Sampling (All Samples)")
agg = []
for r in rows:
    if r and r[0].isdigit() and len(r) > ie:
        try:
            agg.append((int(r[ie]), int(r[ws]), int(r[0]), r[1].strip()[:90]))
        except ValueError:
            pass
T = sum(a[0] for a in agg) or 1
S = sum(a[1] for a in agg) or 1
print(f"total warp instructions {T}, stall samples {S}")
for a in sorted(agg, reverse=True)[:top]:
    print(f"{a[0]/T:6.1%} {a[1]/S:6.1%}  L{a[2]:5d}  {a[3]}")
