"""Diagnostics: per-step overhead of the C2 forward outside the kernel (profiling events on/off,
L2 flush on/off, back-to-back). Prints ms per step for each variant (CUDA events)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_iiswc_lica22_b200 as mg
from workloads import get_config, make_qkv

c = get_config(sys.argv[1] if len(sys.argv) > 1 else "C2")
plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=0)
Q, K, V = (torch.from_numpy(x.view(np.int16)).view(torch.bfloat16).cuda() for x in (q, k, v))
O = torch.empty_like(Q)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
for _ in range(20):
    mg.sparse_attention_fwd(plan, Q, K, V, O, s)
torch.cuda.synchronize()


def run(prof, fl, n=300):
    plan.set_profiling(prof)
    ev = []
    for _ in range(n):
        if fl:
            flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        mg.sparse_attention_fwd(plan, Q, K, V, O, s)
        b.record(s)
        ev.append((a, b))
    torch.cuda.synchronize()
    r = plan.get_profile() if prof else None
    plan.set_profiling(False)
    t = [a.elapsed_time(b) for a, b in ev]
    return np.mean(t), np.median(t), (r["coarse_ms"] / r["calls"] if r else None)


for prof in (True, False):
    for fl in (True, False):
        print(f"profiling={prof} flush={fl}: mean/median/kernel ms", run(prof, fl))
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(s)
for _ in range(300):
    mg.sparse_attention_fwd(plan, Q, K, V, O, s)
e1.record(s)
torch.cuda.synchronize()
print("back-to-back (no flush, no per-step events):", e0.elapsed_time(e1) / 300)
