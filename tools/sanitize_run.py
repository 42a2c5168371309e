"""Small forwards for compute-sanitizer runs (racecheck / synccheck / memcheck): C1, a mixed pattern
with strips, CSR rows (serial and concurrent coarse || fine), split dense-row chunks, padding, a
batched plan and b = 64; each checked against the oracle so a sanitizer-perturbed run still has to
be correct.  Usage: compute-sanitizer --tool racecheck python tools/sanitize_run.py"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import paper_conf_iiswc_lica22_b200 as mg  # noqa: E402
from gpu_util import err_stats, from_device, to_device  # noqa: E402
from oracle import dense_masked_attention, head_inputs_f64  # noqa: E402
from workloads import get_config, make_qkv, random_residual  # noqa: E402


def check(name, plan, q, k, v, window, G, E, lens=None):
    Q, K, V = (to_device(x) for x in (q, k, v))
    if lens is None:
        got = from_device(mg.sparse_attention_fwd(plan, Q, K, V))
    else:
        got = from_device(mg.sparse_attention_fwd_padded(plan, Q, K, V, torch.from_numpy(lens).cuda()))
    worst = 0.0
    for b in range(q.shape[0]):
        for h in range(q.shape[1]):
            Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
            ref = dense_masked_attention(Qh, Kh, Vh, window, G, E, valid_len=None if lens is None else int(lens[b]))
            worst = max(worst, err_stats(got[b, h], ref)[0])
    print(f"{name}: max-abs {worst:.3e}", flush=True)
    assert worst <= 2e-2 * 4


def main():
    c = get_config("C1")
    q, k, v = make_qkv(1, 1, c.L, 64, seed=0)
    check("C1", mg.Plan(c.L, 1, 64, c.window, c.global_idx, c.extra_idx), q, k, v, c.window, c.global_idx, c.extra_idx)
    L, H, W = 512, 2, 128
    G = np.array([0, 1, 130], np.int32)
    E = random_residual(L, W, 4, seed=3)
    q, k, v = make_qkv(1, H, L, 64, seed=5)
    for name, kw in [("mixed/strips", {}), ("mixed/csr", dict(strip_max_cols=-1)),
                     ("mixed/concurrent", dict(strip_max_cols=-1, concurrency=2)), ("mixed/dense-split", dict(dense_chunk=1)),
                     ("mixed/b64", dict(block=64)), ("mixed/few-ctas", dict(num_sms=1, strip_max_cols=-1)),
                     ("mixed/sm-split", dict(strip_max_cols=-1, concurrency=3))]:
        check(name, mg.Plan(L, H, 64, W, G, E, **kw), q, k, v, W, G, E)
    q2, k2, v2 = make_qkv(2, H, L, 64, seed=7)
    check("padded", mg.Plan(L, H, 64, W, G, E), q2, k2, v2, W, G, E, lens=np.array([L, 200], np.int32))
    print("sanitize_run ok")


if __name__ == "__main__":
    main()
