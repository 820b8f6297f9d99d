"""Instruction-executed profile of a kernel's SASS (from an ncu report), bucketed by PC index."""
import csv, io, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
lines = out.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"Address"'))
rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
ins = [int(r["Instructions Executed"] or 0) for r in rows]
T = sum(ins)
print("total warp instructions", T, "sass lines", len(rows))
step = int(sys.argv[2]) if len(sys.argv) > 2 else 200
for a in range(0, len(rows), step):
    s = sum(ins[a:a + step])
    if s / T > 0.01:
        # representative instruction
        k = max(range(a, min(a + step, len(rows))), key=lambda i: ins[i])
        print(f"[{a:5d},{a+step:5d}) {s/T:6.1%}  e.g. #{k} {rows[k]['Source'].strip()[:70]}")
