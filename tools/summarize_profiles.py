"""Summarise ncu captures into profiles/ (run locally after tools/profile_round.sh on the GPU).

    python tools/summarize_profiles.py <round tag, e.g. r01>
Writes profiles/<tag>_launches_<W>.csv (our kernels only), profiles/<tag>_ncu_<name>.txt and
updates profiles/ncu_traffic.json (dram bytes per launch of the dominant kernels).
"""
import csv, io, json, os, subprocess, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
os.makedirs(PROF, exist_ok=True)

WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors.sum",
        "lts__t_sectors.sum.pct_of_peak_sustained_elapsed", "LTS.TriageCompute.lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "lts__t_requests_srcunit_tex.sum",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.per_cycle_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second",
        "l1tex__t_bytes.sum", "smsp__inst_executed.sum"]


def raw(rep):
    r = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(r)))
    return {h: (u, v) for h, u, v in zip(rows[0], rows[1], rows[2])}


traffic_path = os.path.join(PROF, "ncu_traffic.json")
traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
for name, cfg, key in [("full_c2_coarse", "C2", "coarse"), ("full_c4_fine", "C4", "fine"),
                       ("full_c4_coarse", "C4", "coarse"), ("full_c3_coarse", "C3", "coarse"),
                       ("full_c2d128_coarse", "C2-d128", "coarse")]:
    rep = os.path.join(OUT, name + ".ncu-rep")
    if not os.path.exists(rep):
        continue
    m = raw(rep)
    lines = [f"# ncu --set full, {name} ({cfg}), round {tag}; kernel {m.get('Kernel Name', ('', ''))[1][:90]}"]
    for w in WANT:
        if w in m:
            lines.append(f"{w} [{m[w][0]}] = {m[w][1]}")
    open(os.path.join(PROF, f"{tag}_ncu_{name}.txt"), "w").write("\n".join(lines) + "\n")
    def tobytes(u, v):
        f = float(v.replace(",", ""))
        return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
    rd = tobytes(*m["dram__bytes_read.sum"]); wr = tobytes(*m["dram__bytes_write.sum"])
    ent = {"dram_bytes_per_launch": rd + wr, "dram_read": rd, "dram_write": wr,
           "source": f"profiles/{tag}_ncu_{name}.txt"}
    if "lts__t_sectors.sum" in m:
        ent["lts_bytes_per_launch"] = 32.0 * float(m["lts__t_sectors.sum"][1].replace(",", ""))
        ent["lts_sectors_pct_of_peak"] = float(m["lts__t_sectors.sum.pct_of_peak_sustained_elapsed"][1].replace(",", ""))
        ent["l2_hit_rate_pct"] = float(m["lts__t_sector_hit_rate.pct"][1].replace(",", ""))
    traffic.setdefault(cfg, {})[key] = ent
json.dump(traffic, open(traffic_path, "w"), indent=1)
for W in ("C2", "C3", "C4", "C2-d128"):
    src = os.path.join(OUT, f"launches_{W}.csv")
    if not os.path.exists(src):
        continue
    rows = [l for l in open(src) if l.startswith('"ID"') or "mg::" in l or "coarse" in l or "fine_" in l]
    open(os.path.join(PROF, f"{tag}_launches_{W}.csv"), "w").writelines(rows)
print("written", sorted(os.listdir(PROF)))
