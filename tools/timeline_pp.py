"""Per-tile event timeline of the paired-pipeline coarse kernel (diagnostics; needs a GPU and an
MG_TIMELINE=1 build: MG_TIMELINE=1 python -m paper_conf_iiswc_lica22_b200.build).

    python tools/timeline_pp.py [C2] [--dump CTA]

Fields per tile (coarse_pp_sm100.cu tl_rec): 0 softmax S(n)+V(n) ready, 1 softmax P.V(n-1) done,
2 softmax P(n) stored, 3 MMA S(n) issued, 4 MMA P.V(n) issued, 5 producer K(n) issued,
6 producer V(n) issued. Prints mean intervals over all CTAs and the raw timeline of one CTA.
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_iiswc_lica22_b200 as mg  # noqa: E402
from workloads import get_config, make_qkv  # noqa: E402

T = 128


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    name = args[0] if args else "C2"
    dump = int(sys.argv[sys.argv.index("--dump") + 1]) if "--dump" in sys.argv else 0
    c = get_config(name)
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=0)
    Q, K, V = (torch.from_numpy(x.view(np.int16)).view(torch.bfloat16).cuda() for x in (q, k, v))
    for _ in range(3):
        mg.sparse_attention_fwd(plan, Q, K, V)
    ncta = 2 * torch.cuda.get_device_properties(0).multi_processor_count
    buf = torch.zeros(256 + 4 * T * ncta, dtype=torch.int64, device="cuda")
    plan.set_trace(buf)
    mg.sparse_attention_fwd(plan, Q, K, V)
    torch.cuda.synchronize()
    plan.set_trace(None)
    rec = buf.cpu().numpy()[256:].view(np.uint32).reshape(ncta, T, 8).astype(np.int64)
    smid = rec[:, 0, 7].copy()
    rec[:, 0, 7] = 0
    d = lambda a, b: (b - a + 2**31) % 2**32 - 2**31   # wrap-safe difference of 32-bit clocks
    iv = {
        "softmax: S(n) ready -> P.V(n-1) done": [],
        "softmax: P.V(n-1) done -> P(n) stored": [],
        "softmax: P(n) stored -> S(n+1) ready": [],
        "MMA: P(n) stored -> P.V(n) issued": [],
        "MMA: S(n+1) issued -> softmax S(n+1) ready": [],
        "MMA: P.V(n-1) issued -> softmax sees P.V(n-1) done": [],
        "producer: K(n) issued -> MMA S(n) issued": [],
        "producer: V(n) issued -> MMA P.V(n) issued": [],
        "tile period (S ready n -> n+1)": [],
    }
    for cta in range(ncta):
        r = rec[cta]
        nt = int(np.count_nonzero(r[:, 2]))
        for n in range(1, nt - 1):
            e, f = r[n], r[n + 1]
            iv["softmax: S(n) ready -> P.V(n-1) done"].append(d(e[0], e[1]))
            iv["softmax: P.V(n-1) done -> P(n) stored"].append(d(e[1], e[2]))
            iv["softmax: P(n) stored -> S(n+1) ready"].append(d(e[2], f[0]))
            iv["MMA: P(n) stored -> P.V(n) issued"].append(d(e[2], e[4]))
            iv["MMA: S(n+1) issued -> softmax S(n+1) ready"].append(d(f[3], f[0]))
            iv["MMA: P.V(n-1) issued -> softmax sees P.V(n-1) done"].append(d(r[n - 1][4], e[1]))
            iv["producer: K(n) issued -> MMA S(n) issued"].append(d(e[5], e[3]))
            iv["producer: V(n) issued -> MMA P.V(n) issued"].append(d(e[6], e[4]))
            iv["tile period (S ready n -> n+1)"].append(d(e[0], f[0]))
    for k_, v_ in iv.items():
        a = np.array(v_)
        print(f"{k_:55s} mean {a.mean():8.0f}  median {np.median(a):8.0f}  p90 {np.percentile(a, 90):8.0f}")
    same = np.nonzero(smid == smid[dump])[0]
    print(f"CTA {dump} on SM {smid[dump]} (CTAs on that SM: {list(same)})")
    base = rec[dump, 0, 5]
    print("  n   S_rdy  pv_dn  P_st  | S_iss  PV_iss | K_iss  V_iss")
    for n in range(min(40, T)):
        e = rec[dump, n]
        if not e[2]:
            break
        print(f"{n:3d} " + " ".join(f"{d(base, x):6d}" for x in e[:3]) + " | " +
              " ".join(f"{d(base, x):6d}" for x in e[3:5]) + " | " + " ".join(f"{d(base, x):6d}" for x in e[5:7]))


if __name__ == "__main__":
    main()
