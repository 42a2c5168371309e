"""Stall-reason totals per warp-role region of a kernel in an .ncu-rep: regions start at each
USETMAXREG (role entry) in SASS order. Usage: ncu_regions.py rep"""
import csv, io, subprocess, sys
rep = sys.argv[1]
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h = rows[1]; data = rows[2:]
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
ci = [h.index(c) for c in cols]
i_src, i_s, i_ex = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
regions, cur = [], None
for x in data:
    s = x[i_src]
    if "USETMAXREG" in s or cur is None:
        cur = {"start": x[0], "first": s.strip()[:40], "tot": 0, "ex": 0, "st": [0]*len(cols), "marks": set()}
        regions.append(cur)
    for m in ("UTMALDG", "UTCHMMA", "MUFU.EX2", "LDTM", "ATOMG", "STG", "UTMAPF"):
        if m in s: cur["marks"].add(m)
    v = int(x[i_s]) if x[i_s].isdigit() else 0
    cur["tot"] += v
    cur["ex"] += int(x[i_ex]) if x[i_ex].isdigit() else 0
    for k, j in enumerate(ci):
        cur["st"][k] += int(x[j]) if x[j].isdigit() else 0
for r in regions:
    top = sorted(zip(cols, r["st"]), key=lambda t: -t[1])[:6]
    print(f"{r['start']} {r['first']:40s} samples {r['tot']:6d} inst {r['ex']:10d} marks {sorted(r['marks'])}")
    print("      ", ", ".join(f"{c[6:]} {v}" for c, v in top))
