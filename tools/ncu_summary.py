"""Summarise an .ncu-rep: key raw metrics + top stalled SASS lines. Usage: ncu_summary.py rep [ntop]"""
import csv, io, subprocess, sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units = rows[0], rows[1]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_xu.avg.pct",
        "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread", "smsp__inst_executed.sum",
        "sm__cycles_elapsed.avg", "smsp__average_warps_issue_stalled", "sm__throughput.avg.pct",
        "smsp__issue_active.avg.pct", "sm__pipe_fma_cycles_active.avg.pct", "sm__pipe_alu_cycles_active.avg.pct",
        "l1tex__data_bank_conflicts", "smsp__inst_executed_pipe_uniform"]
for r in rows[2:]:
    print("== kernel:", r[hdr.index("Kernel Name")][:80] if "Kernel Name" in hdr else "")
    for h, u, v in zip(hdr, units, r):
        if any(h.startswith(w) for w in want) and not h.endswith(".max") and not h.endswith(".min"):
            if "stalled" in h and ("_not_issued" in h or float(v or 0) < 0.05):
                continue
            print(f"  {h} [{u}] = {v}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
srows = list(csv.reader(io.StringIO(src)))
h2 = srows[1]
data = srows[2:]
i_s, i_src, i_ex = h2.index("Warp Stall Sampling (All Samples)"), h2.index("Source"), h2.index("Instructions Executed")
tot = sum(int(x[i_s]) for x in data if x[i_s].isdigit())
print("== stall samples", tot)
for x in sorted(data, key=lambda x: -int(x[i_s]) if x[i_s].isdigit() else 0)[:ntop]:
    print(f"  {x[i_s]:>6} {x[i_ex]:>8} {x[0][-5:]} {x[i_src][:100]}")
