"""Print SASS lines of an .ncu-rep with stall samples and execution counts, optionally only
around lines matching a regex: ncu_sass_window.py rep [regex] [context]"""
import csv, io, re, subprocess, sys

rep = sys.argv[1]
pat = re.compile(sys.argv[2]) if len(sys.argv) > 2 else None
ctx = int(sys.argv[3]) if len(sys.argv) > 3 else 6
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h = rows[1]
data = rows[2:]
i_s, i_src, i_ex = h.index("Warp Stall Sampling (All Samples)"), h.index("Source"), h.index("Instructions Executed")
keep = set()
for k, x in enumerate(data):
    if pat is None or pat.search(x[i_src]):
        keep.update(range(max(0, k - ctx), min(len(data), k + ctx + 1)))
last = -2
for k in sorted(keep):
    if k != last + 1:
        print("   ...")
    x = data[k]
    print(f"{x[i_s]:>6} {x[i_ex]:>8} {x[0][-5:]} {x[i_src][:110]}")
    last = k
