"""Aggregate an .ncu-rep's per-SASS stall samples by CUDA source line, using the line table of a
locally built cubin of the same source (nvdisasm -g). Usage:
    ncu_lines.py rep.ncu-rep kernel.cubin mangled-kernel-substring [ntop]"""
import collections, csv, io, re, subprocess, sys

rep, cubin, kname = sys.argv[1:4]
ntop = int(sys.argv[4]) if len(sys.argv) > 4 else 40
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h = rows[1]
data = rows[2:]
i_s, i_src, i_ex = h.index("Warp Stall Sampling (All Samples)"), h.index("Source"), h.index("Instructions Executed")
base = int(data[0][0], 16)
samples = {int(x[0], 16) - base: (int(x[i_s] or 0), int(x[i_ex] or 0), x[i_src]) for x in data}
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
lines = {}
cur = None
infn = False
for l in dis.split("\n"):
    if l.startswith(".text.") or "Function :" in l or l.strip().startswith(".section"):
        infn = kname in l
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (m.group(1).split("/")[-1], int(m.group(2)))
    m2 = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m2 and infn:
        lines[int(m2.group(1), 16)] = cur
agg = collections.Counter()
ex = collections.Counter()
miss = 0
for off, (s, e, _) in samples.items():
    key = lines.get(off)
    if key is None:
        miss += s
        continue
    agg[key] += s
    ex[key] = max(ex[key], e)
tot = sum(agg.values()) + miss
print(f"total samples {tot} (unmapped {miss}); mapped {len(lines)} SASS lines")
srcfiles = {}
for (f, ln), s in agg.most_common(ntop):
    path = [p for p in ["paper_conf_iiswc_lica22_b200/csrc/" + f] ]
    try:
        text = srcfiles.setdefault(f, open(path[0]).read().split("\n"))[ln - 1].strip()
    except Exception:
        text = ""
    print(f"{s:>6} {100*s/tot:5.1f}% {f}:{ln:<5} exec={ex[(f, ln)]:>8}  {text[:90]}")
