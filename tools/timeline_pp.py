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
F = 24   # fields per tile (coarse_pp_sm100.cu kTlF)


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
    buf = torch.zeros(256 + (12 * T + 128) * ncta, dtype=torch.int64, device="cuda")
    plan.set_trace(buf)
    mg.sparse_attention_fwd(plan, Q, K, V)
    torch.cuda.synchronize()
    plan.set_trace(None)
    raw = buf.cpu().numpy()[256:].view(np.uint32).astype(np.int64)
    rec = raw[:ncta * T * F].reshape(ncta, T, F)
    itm = raw[ncta * T * F:ncta * T * F + ncta * 256].reshape(ncta, 32, 8)
    smid = rec[:, 0, 15].copy()
    rec[:, 0, 15] = 0
    d = lambda a, b: (b - a + 2**31) % 2**32 - 2**31   # wrap-safe difference of 32-bit clocks
    iv = {}
    def add(k, v):
        iv.setdefault(k, []).append(v)
    for cta in range(ncta):
        r = rec[cta]
        nt = int(np.count_nonzero(r[:, 2]))
        for n in range(1, nt - 1):
            e, f = r[n], r[n + 1]
            last_p = max(e[2], e[8], e[9], e[10], key=lambda x: d(e[2], x))
            add("softmax: S(n) ready -> P.V(n-1) done", d(e[0], e[1]))
            add("softmax: P.V(n-1) done -> P(n) stored (warp 0)", d(e[1], e[2]))
            add("softmax: warp skew, last P(n) - warp 0 P(n)", d(e[2], last_p))
            add("softmax: P(n) stored (last warp) -> S(n+1) ready", d(last_p, f[0]))
            add("MMA: last P(n) stored -> MMA sees p_full(n)", d(last_p, e[7]))
            add("MMA: sees p_full(n) -> P.V(n) MMAs issued", d(e[7], e[4]))
            add("MMA: P.V(n) issued -> softmax sees P.V(n) done", d(e[4], f[1]))
            add("MMA: k_full(n+1) seen -> S(n+1) issued", d(f[14], f[3]))
            add("MMA: S(n+1) issued -> softmax S(n+1) ready", d(f[3], f[0]))
            add("producer: K(n) issued -> MMA sees k_full(n)", d(e[5], e[14]))
            add("tile period (S ready n -> n+1)", d(e[0], f[0]))
            add("softmax: S(n) ready -> S in registers", d(e[0], e[16]))
            add("softmax: S in registers -> exps done", d(e[16], e[17]))
            add("softmax: exps done -> P.V(n-1) done (wait)", d(e[17], e[1]))
            add("softmax: S(n+1) complete when P(n) stored (fraction)", int(e[18]))
            if e[11]:
                add("epilogue: start -> last P.V done + O read", d(e[11], e[12]))
                add("epilogue: O read -> end", d(e[12], e[13]))
                add("epilogue end -> next S ready", d(e[13], f[0]))
    for k_, v_ in iv.items():
        a = np.array(v_)
        print(f"{k_:55s} n {len(a):6d} mean {a.mean():7.0f} median {np.median(a):7.0f} p90 {np.percentile(a, 90):7.0f}")
    # kernel span per CTA (first producer event to last epilogue end)
    spans = []
    for cta in range(ncta):
        r = rec[cta]
        nt = int(np.count_nonzero(r[:, 2]))
        if nt:
            spans.append(d(r[0, 5], max(r[:nt, 13].max(), r[:nt, 2].max())))
    print("CTA spans (first 128 tiles): median", int(np.median(spans)), "max", int(np.max(spans)))
    base = rec[dump, 0, 5]
    print(" it  sch_free sch_pub  prod_it  prod_Q  prod_tr |   smx_it  mma_it  mma_Q")
    for i in range(12):
        e = itm[dump, i]
        if not e[2]:
            break
        f = lambda x: f"{d(base, x):8d}" if x else "       -"
        print(f"{i:3d} " + " ".join(f(x) for x in e[:5]) + " | " + " ".join(f(x) for x in e[5:8]))
    same = np.nonzero(smid == smid[dump])[0]
    print(f"CTA {dump} on SM {smid[dump]} (CTAs on that SM: {[int(x) for x in same]})")
    base = rec[dump, 0, 5]
    print("  n   S_rdy  pv_dn   P_st0  P_last | K_seen  S_iss  pfull  PV_iss | K_iss  V_iss | epi_s  epi_o  epi_e")
    for n in range(min(48, T)):
        e = rec[dump, n]
        if not e[2]:
            break
        last_p = max(e[2], e[8], e[9], e[10], key=lambda x: d(e[2], x))
        f = lambda x: f"{d(base, x):7d}" if x else "      -"
        print(f"{n:3d} " + " ".join(f(x) for x in (e[0], e[1], e[2], last_p)) + " | " +
              " ".join(f(x) for x in (e[14], e[3], e[7], e[4])) + " | " + " ".join(f(x) for x in e[5:7]) + " | " +
              " ".join(f(x) for x in e[11:14]))


if __name__ == "__main__":
    main()
