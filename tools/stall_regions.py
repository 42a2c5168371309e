"""Stall-reason totals of an ncu source-page CSV (--page source --csv --print-source sass), overall
and per code region (region boundaries = SASS lines matching a marker instruction).

    python tools/stall_regions.py gpurun_out/stall_c2_source.csv
"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = rows[2:]
cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
isrc = hdr.index("Source")
tot = {hdr[i]: 0 for i in cols}
for r in data:
    for i in cols:
        try:
            tot[hdr[i]] += int(r[i])
        except ValueError:
            pass
s = sum(tot.values())
print("all samples", s)
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    if v:
        print(f"  {k:22s} {v:8d} {100.0 * v / s:5.1f}%")
# top 40 instructions by samples with their dominant reason
ranked = []
for n, r in enumerate(data):
    try:
        smp = int(r[hdr.index("Warp Stall Sampling (All Samples)")])
    except ValueError:
        continue
    reasons = sorted(((int(r[i]) if r[i].isdigit() else 0, hdr[i]) for i in cols), reverse=True)[:2]
    ranked.append((smp, n, r[isrc].strip()[:60], reasons))
ranked.sort(reverse=True)
print("top instructions (samples, sass line, instr, top reasons):")
for smp, n, src, reasons in ranked[:int(sys.argv[2]) if len(sys.argv) > 2 else 40]:
    print(f"  {smp:6d} {n:6d} {src:60s} {reasons}")
