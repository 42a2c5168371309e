"""Debug: global rows of every (b, h) vs the oracle; prints the bad (b, h) list."""
import os, sys
import numpy as np
import torch
R = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path[:0] = [R, os.path.join(R, "tests")]
import paper_conf_iiswc_lica22_b200 as mg
from oracle import attention_rows, global_flags, ExtraIndex, head_inputs_f64
from workloads import get_config, make_qkv
from gpu_util import from_device, to_device

c = get_config(sys.argv[1] if len(sys.argv) > 1 else "C2")
q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=c.seed)
plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
Q, K, V = (to_device(x, "bf16") for x in (q, k, v))
g = global_flags(c.L, c.global_idx); ex = ExtraIndex(c.L, c.extra_idx)
rows = np.asarray(c.global_idx)
refs = {}
for rep in range(3):
    got = from_device(mg.sparse_attention_fwd(plan, Q, K, V))
    bad = []
    for b in range(c.B):
        for h in range(c.H):
            if (b, h) not in refs:
                Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
                refs[(b, h)] = attention_rows(Qh, Kh, Vh, rows, c.window, g, ex)
            e = np.abs(got[b, h, rows] - refs[(b, h)]).max()
            if e > 2e-2:
                bad.append((b, h, round(float(e), 3)))
    print("rep", rep, "bad", bad)
