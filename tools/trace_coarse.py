"""Read the coarse kernel's warp-role timeline for CTA 0 (diagnostics; needs a GPU).

    python tools/trace_coarse.py [C2] [--dump N]

Prints, per role, the mean cycles spent between consecutive events, which shows which
barrier each warp role waits on (producer: kv_empty; MMA: K ready / O buffer free / P ready;
softmax: S ready / P stored / O consumed).
"""
import os
import sys
from collections import defaultdict

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_iiswc_lica22_b200 as mg  # noqa: E402
from workloads import get_config, make_qkv  # noqa: E402

NAMES = {(0, 1): "P:item", (0, 2): "P:qfree", (0, 3): "P:kvfree", (0, 4): "P:slotwait", (0, 5): "P:slotfree",
         (1, 0): "M:qready", (1, 1): "M:kready", (1, 2): "M:Sissue", (1, 4): "M:Pready", (1, 5): "M:PVissue",
         (2, 1): "S:tile", (2, 2): "S:Sready", (2, 3): "S:Pstored", (2, 4): "S:Oconsumed", (2, 5): "S:itemO",
         (2, 6): "S:xch", (2, 7): "S:ld0", (2, 8): "S:max0", (2, 9): "S:pvwait0", (2, 10): "S:exp0",
         (2, 11): "S:ld1", (2, 12): "S:max1", (2, 13): "S:pvwait1", (2, 14): "S:exp1", (3, 1): "T:tile", (3, 2): "T:Sready", (3, 3): "T:Pstored", (3, 4): "T:Oconsumed",
         (3, 5): "T:itemO", (3, 6): "T:xch",
         (3, 7): "T:ld0", (3, 8): "T:max0", (3, 9): "T:pvwait0", (3, 10): "T:exp0",
         (3, 11): "T:ld1", (3, 12): "T:max1", (3, 13): "T:pvwait1", (3, 14): "T:exp1"}


def main():
    name = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("-") else "C2"
    dump = int(sys.argv[sys.argv.index("--dump") + 1]) if "--dump" in sys.argv else 60
    c = get_config(name)
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=0)
    Q, K, V = (torch.from_numpy(x.view(np.int16)).view(torch.bfloat16).cuda() for x in (q, k, v))
    for _ in range(3):
        mg.sparse_attention_fwd(plan, Q, K, V)
    buf = torch.zeros((1 << 16, 2), dtype=torch.int64, device="cuda")
    plan.set_trace(buf)
    mg.sparse_attention_fwd(plan, Q, K, V)
    torch.cuda.synchronize()
    plan.set_trace(None)
    t = buf.cpu().numpy().view(np.uint64)
    seg = t.shape[0] // 4
    parts = []
    for r in range(4):
        s_ = t[r * seg:(r + 1) * seg]
        parts.append(s_[1:int(s_[0, 0]) + 1])
    ev = np.concatenate(parts)
    n = len(ev)
    order = np.argsort(ev[:, 0], kind="stable")
    ev = ev[order]
    t0 = ev[0, 0]
    last = {}
    gaps = defaultdict(list)
    for i, (clk, code) in enumerate(ev):
        role, e, arg = int(code >> 56), int((code >> 48) & 0xFF), int(code & 0xFFFFFFFFFFFF)
        key = (min(role, 2), e) if role != 3 else (3, e)
        if role in last:
            pk, pclk = last[role]
            gaps[(NAMES.get(pk, pk), NAMES.get(key, key))].append(int(clk - pclk))
        last[role] = (key, clk)
        if i < dump:
            print(f"{int(clk - t0):>9}  {NAMES.get(key, key):<12} {arg}")
    print(f"\n{n} events, span {int(ev[-1, 0] - t0)} cycles")
    print("mean cycles between consecutive events of the same role:")
    for (a, b), v_ in sorted(gaps.items(), key=lambda x: -sum(x[1])):
        print(f"  {str(a):<12} -> {str(b):<12} n={len(v_):>5} mean={np.mean(v_):>8.1f} total={sum(v_):>10}")


if __name__ == "__main__":
    main()
