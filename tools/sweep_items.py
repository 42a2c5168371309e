"""Per-item vs per-tile cost of the coarse kernel (diagnostics; needs a GPU).

    python tools/sweep_items.py

Times the forward (CUDA events, L2 flushed) on band-only synthetic configs (no global rows, no
CSR residual) with different windows, so the number of tiles per item varies while the number of
items stays fixed, and fits time = a * items + b * tiles by least squares.
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_iiswc_lica22_b200 as mg  # noqa: E402
from workloads import make_qkv  # noqa: E402


def time_cfg(L, window, B, H, G=0, reps=50):
    glob = np.arange(G, dtype=np.int32) * (L // max(G, 1)) if G else np.zeros(0, np.int32)
    plan = mg.Plan(L, H, 64, window, glob, np.zeros(0, np.int32))
    info = plan.info()
    q, k, v = make_qkv(B, H, L, 64, seed=0)
    Q, K, V = (torch.from_numpy(x.view(np.int16)).view(torch.bfloat16).cuda() for x in (q, k, v))
    O = torch.empty_like(Q)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    ts = []
    for i in range(reps + 5):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        mg.sparse_attention_fwd(plan, Q, K, V, O)
        e1.record()
        torch.cuda.synchronize()
        if i >= 5:
            ts.append(e0.elapsed_time(e1) * 1e3)
    BH = B * H
    tiles = info["n_tiles"] * BH + 0
    items = info["n_items"] * BH
    return np.median(ts), items, tiles, info


def main():
    rows = []
    for window in (128, 256, 512, 1024, 2048):
        t, items, tiles, info = time_cfg(4096, window, 8, 12)
        rows.append((t, items, tiles))
        print(f"L=4096 w={window:>5}: {t:8.1f} us  items {items:>6}  tiles {tiles:>7}  "
              f"({tiles / items:.1f} tiles/item)  ns/tile/SM {t * 1e3 * 148 / tiles:7.1f}")
    A = np.array([[r[1], r[2]] for r in rows], dtype=float)
    y = np.array([r[0] for r in rows])
    (a, b), *_ = np.linalg.lstsq(A, y, rcond=None)
    print(f"fit: {a * 148 * 1e3:.0f} ns per item per SM, {b * 148 * 1e3:.0f} ns per tile per SM "
          f"({a * 148 * 1965:.0f} / {b * 148 * 1965:.0f} cycles)")


if __name__ == "__main__":
    main()
