"""Bucket an ncu report's per-instruction counts and stall samples by k_dp_hld phase (source line ranges)."""
import csv, io, re, subprocess, sys
rep = sys.argv[1]
src = sys.argv[2] if len(sys.argv) > 2 else "paper_conf_date_liulzclly22_b200/csrc/dp_hld.cu"
text = open(src).read().split("\n")
marks = []
for i, l in enumerate(text, 1):
    m = re.search(r"// ---- (P\d)|// (P3[ab]|P4b)", l)
    if m:
        marks.append((i, m.group(1) or m.group(2)))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
agg = {}
cur_file = None
hdr = None
for r in rows:
    if r and r[0] in ("File Name", "File Path"):
        cur_file = r[1] if len(r) > 1 else None
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if not r or not r[0].isdigit() or hdr is None:
        continue
    ie = hdr.index("Instructions Executed"); ws = hdr.index("Warp Stall Sampling (All Samples)")
    try:
        n = int(r[ie]); s = int(r[ws])
    except (ValueError, IndexError):
        continue
    line = int(r[0])
    if cur_file and cur_file.endswith("dp_hld.cu"):
        ph = "pre"
        for (ln, name) in marks:
            if line >= ln:
                ph = name
        if line < marks[0][0]:
            ph = "helpers(L%d)" % (line // 20 * 20)
    else:
        ph = (cur_file or "?").split("/")[-1]
    a = agg.setdefault(ph, [0, 0, {}])
    a[0] += n; a[1] += s
    for j, name in enumerate(hdr):
        if name.startswith("stall_") and "Not Issued" not in name and j < len(r):
            try:
                a[2][name[6:]] = a[2].get(name[6:], 0) + int(r[j])
            except ValueError:
                pass
T = sum(a[0] for a in agg.values()) or 1
S = sum(a[1] for a in agg.values()) or 1
for k, (n, s, st) in sorted(agg.items(), key=lambda x: -x[1][1]):
    top = sorted(st.items(), key=lambda x: -x[1])[:4]
    tot = sum(st.values()) or 1
    print(f"{k:22s} inst {n:9d} {n/T:6.1%}   stall samples {s:7d} {s/S:6.1%}  " + ", ".join(f"{a}={b/tot:.0%}" for a, b in top))
