"""Per-phase cycle breakdown of the coarse kernel's warp roles (diagnostics; needs a GPU and a
build with MG_TRACE=1, see tools/trace_run.sh).

    python tools/trace_coarse.py [C2]

Each profiled warp (producer, MMA issuer, softmax warps 4 and 8) charges the cycles between
consecutive marks to a phase; the kernel adds the per-CTA counters to a device buffer at exit.
Prints the mean cycles per CTA spent in each phase and its share of the role's total.
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_iiswc_lica22_b200 as mg  # noqa: E402
from workloads import get_config, make_qkv  # noqa: E402

PHASES = {
    0: ("producer", ["item wait", "q_empty wait", "Q load/gather", "kv_empty wait", "K/V TMA issue",
                     "strip gather"]),
    1: ("mma", ["item wait", "q_full wait", "kv_full wait", "-", "S issue", "o_free wait",
                "p_full wait", "PV issue", "-", "-"]),
    2: ("softmax g0", ["item wait+meta", "-", "s_full wait", "tmem ld S", "max+decide",
                       "O rescale", "-", "exp+P store", "p_full arrive", "epi pv wait+xch",
                       "epi O ld+o_free", "epi store"]),
}
PHASES[3] = ("softmax g1", PHASES[2][1])


def main():
    name = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("-") else "C2"
    c = get_config(name)
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=0)
    Q, K, V = (torch.from_numpy(x.view(np.int16)).view(torch.bfloat16).cuda() for x in (q, k, v))
    for _ in range(3):
        mg.sparse_attention_fwd(plan, Q, K, V)
    buf = torch.zeros((8, 16), dtype=torch.int64, device="cuda")
    plan.set_trace(buf)
    mg.sparse_attention_fwd(plan, Q, K, V)
    torch.cuda.synchronize()
    plan.set_trace(None)
    t = buf.cpu().numpy()
    print(f"workload {name}, debug flags {os.environ.get('MG_DEBUG_FLAGS', '0')}")
    for role, (rname, phases) in PHASES.items():
        ncta = max(int(t[role, 15]), 1)
        tot = t[role, :12].sum() / ncta
        print(f"{rname:<11} ({ncta} CTAs) total {tot:10.0f} cycles/CTA")
        for k_, ph in enumerate(phases):
            cyc = t[role, k_] / ncta
            print(f"    {ph:<22} {cyc:10.0f}  {100 * cyc / max(tot, 1):5.1f}%")


if __name__ == "__main__":
    main()
