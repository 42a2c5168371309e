"""Per-item event timeline of the coarse kernel (diagnostics; needs a GPU and an MG_TIMELINE=1
build, see tools/trace_run.sh).

    python tools/timeline_coarse.py [C2]

Every CTA records, per item, the SM clock at: 0 softmax item start, 1 first S ready, 2 last P
stored, 3/4 epilogue start/end (run during the next item), 5 MMA Q ready, 6 MMA first S issued,
7 MMA first P.V issued. Prints the mean of the intervals that make up an item boundary.
"""
import os
import sys
from collections import defaultdict

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_iiswc_lica22_b200 as mg  # noqa: E402
from workloads import get_config, make_qkv  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("-") else "C2"
    c = get_config(name)
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=0)
    Q, K, V = (torch.from_numpy(x.view(np.int16)).view(torch.bfloat16).cuda() for x in (q, k, v))
    for _ in range(3):
        mg.sparse_attention_fwd(plan, Q, K, V)
    ncta = torch.cuda.get_device_properties(0).multi_processor_count
    buf = torch.zeros(256 + 8 * 64 * ncta, dtype=torch.int64, device="cuda")
    plan.set_trace(buf)
    mg.sparse_attention_fwd(plan, Q, K, V)
    torch.cuda.synchronize()
    plan.set_trace(None)
    rec = buf.cpu().numpy()[256:].view(np.uint32).reshape(ncta, 64, 16).astype(np.int64)
    iv = defaultdict(list)
    names = {
        "item (start k -> start k+1)": (0, 0, 1),
        "S ready wait (item start -> first S ready)": (0, 1, 0),
        "tiles (first S ready -> last P stored)": (1, 2, 0),
        "last P (k) -> first S ready (k+1)": (2, 1, 1),
        "last P (k) -> epilogue(k) start": (2, 3, 0),
        "epilogue duration": (3, 4, 0),
        "  epi: start -> (m,l) exchanged": (3, 8, 0),
        "  epi: exchanged -> last P.V done": (8, 9, 0),
        "  epi: last P.V done -> O read + o_free": (9, 10, 0),
        "  epi: O read -> stores issued": (10, 4, 0),
        "epilogue end (k) -> last P (k+1)": (4, 2, 1),
        "MMA: Q ready -> first S issued": (5, 6, 0),
        "MMA: first S issued -> first PV issued": (6, 7, 0),
        "MMA: first S issued (k) -> (k+1)": (6, 6, 1),
        "MMA Q ready -> softmax first S ready": (5, 1, 0),
        "softmax last P (k) -> MMA Q ready (k+1)": (2, 5, 1),
        "softmax item start (k+1) -> MMA Q ready (k+1)": (0, 5, 0),
        "MMA first S issued (k+1) -> softmax first S ready (k+1)": (6, 1, 0),
    }
    for cta in range(ncta):
        r = rec[cta]
        n = int(np.count_nonzero(r[:, 0]))
        for kk in range(n - 1):
            for label, (fa, fb, d) in names.items():
                a, b = r[kk, fa], r[kk + d, fb]
                if a and b:
                    dlt = (b - a) & 0xFFFFFFFF
                    iv[label].append(dlt - (1 << 32) if dlt >= 1 << 31 else dlt)
    print(f"workload {name}: mean cycles per item boundary interval (all CTAs)")
    for label in names:
        v = np.array(iv[label])
        if len(v):
            print(f"  {label:<45} mean {v.mean():9.0f}  p50 {np.median(v):9.0f}  p90 {np.percentile(v, 90):9.0f}")


if __name__ == "__main__":
    main()
