"""Debug: C2 forward vs oracle rows of (b, h) = (0, 0): report which rows are off."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
import paper_conf_iiswc_lica22_b200 as mg
from oracle import attention_rows, global_flags, ExtraIndex, head_inputs_f64
from workloads import get_config, make_qkv
from gpu_util import from_device, to_device

c = get_config(sys.argv[1] if len(sys.argv) > 1 else "C2")
q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=c.seed)
plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
Q, K, V = (to_device(x, "bf16") for x in (q, k, v))
got = from_device(mg.sparse_attention_fwd(plan, Q, K, V))
g = global_flags(c.L, c.global_idx); ex = ExtraIndex(c.L, c.extra_idx)
for (b, h) in [(0, 0), (c.B - 1, c.H - 1)]:
    Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
    rows = np.arange(c.L)
    ref = attention_rows(Qh, Kh, Vh, rows, c.window, g, ex)
    e = np.abs(got[b, h] - ref).max(axis=1)
    bad = np.nonzero(e > 2e-2)[0]
    print((b, h), "max", e.max(), "bad rows", len(bad), bad[:40], "blocks", np.unique(bad // 128)[:40])
