"""GPU parity at head dimension d = 128 (D_h is a model parameter).

The coarse kernel runs one CTA per SM at d = 128 (Q/K/V tiles of two 64-column SWIZZLE_128B
sub-tiles, S = Q K^T over 8 K-steps, P.V as two N = 64 halves into 128 TMEM columns of O), the
fine kernel gathers 256-byte rows (16 lanes per row). Every element is compared with the fp64
oracle (O-4) at the north_star bar; the scale is 1/sqrt(128) (A1).
"""
import numpy as np
import pytest
import torch

import paper_conf_iiswc_lica22_b200 as mg
from oracle import ExtraIndex, attention_rows, dense_masked_attention, global_flags, head_inputs_f64
from workloads import get_config, make_qkv, random_residual
from gpu_util import TOL_MAX, TOL_MEAN, err_stats, from_device, to_device

pytestmark = pytest.mark.gpu

D = 128


def oracle_all(q, k, v, window, G, E, lens=None, dtype="bf16"):
    out = np.zeros(q.shape)
    for b in range(q.shape[0]):
        for h in range(q.shape[1]):
            Q, K, V = head_inputs_f64(q, k, v, b, h, dtype)
            g = G[b] if isinstance(G, list) else G
            e = E[b] if isinstance(E, list) else E
            out[b, h] = dense_masked_attention(Q, K, V, window, g, e, valid_len=None if lens is None else int(lens[b]))
    return out


def check(got, ref):
    mx, mean = err_stats(got, ref)
    assert np.isfinite(got).all()
    assert mx <= TOL_MAX * max(1.0, np.abs(ref).max() / 4) and mean <= TOL_MEAN, (mx, mean)


L, H, B, W = 1024, 3, 2, 128
G = np.array([0, 1, 2, 130, 777], np.int32)


def test_c1_pattern_d128():
    c = get_config("C1")
    q, k, v = make_qkv(1, 2, c.L, D, seed=0)
    plan = mg.Plan(c.L, 2, D, c.window, c.global_idx, c.extra_idx)
    check(from_device(mg.sparse_attention_fwd(plan, *(to_device(x) for x in (q, k, v)))),
          oracle_all(q, k, v, c.window, c.global_idx, c.extra_idx))


@pytest.mark.parametrize("kw", [{}, dict(strip_max_cols=-1), dict(strip_max_cols=-1, concurrency=2),
                                dict(dense_chunk=2), dict(force_all_fine=True), dict(block=64),
                                dict(num_sms=2, strip_max_cols=-1), dict(strip_max_cols=-1, fine_kernel=1)],
                         ids=["strips", "csr_rows", "concurrent", "dense_split", "all_fine", "b64", "few_ctas", "ck"])
def test_mixed_pattern_d128(kw):
    E = random_residual(L, W, 6, seed=3)
    q, k, v = make_qkv(B, H, L, D, seed=5, dist="adversarial", global_idx=G)
    plan = mg.Plan(L, H, D, W, G, E, **kw)
    Q, K, V = (to_device(x) for x in (q, k, v))
    ref = oracle_all(q, k, v, W, G, E)
    for _ in range(2):
        check(from_device(mg.sparse_attention_fwd(plan, Q, K, V)), ref)


@pytest.mark.parametrize("dtype", ["bf16", "fp16"])
def test_fine_rows_all_lengths_d128(dtype):
    Lr, Gr = 768, np.array([700], np.int32)
    rng = np.random.default_rng(11)
    pairs = []
    for r in range(Lr):
        n = 1 + r % 70
        pairs += [(r, c) for c in rng.choice(Lr, n, replace=False)]
    E = np.array(pairs, np.int32)
    q, k, v = make_qkv(1, 2, Lr, D, seed=12, dtype=dtype)
    for all_fine in (True, False):
        plan = mg.Plan(Lr, 2, D, 32, Gr, E, strip_max_cols=-1, force_all_fine=all_fine)
        got = from_device(mg.sparse_attention_fwd(plan, *(to_device(x, dtype) for x in (q, k, v))))
        check(got, oracle_all(q, k, v, 32, Gr, E, dtype=dtype))


def test_padded_batched_and_layout_d128():
    Gs = [np.array([0, 5, 700], np.int32), np.array([300], np.int32), np.zeros(0, np.int32),
          np.arange(0, 40, dtype=np.int32)]
    Es = [random_residual(L, W, b + 1, seed=60 + b) for b in range(4)]
    plan = mg.BatchedPlan(L, 2, D, W, Gs, Es)
    q, k, v = make_qkv(4, 2, L, D, seed=52)
    Q, K, V = (to_device(x) for x in (q, k, v))
    lens = np.array([L, 333, 1000, 129], np.int32)
    got = from_device(mg.sparse_attention_fwd_padded(plan, Q, K, V, torch.from_numpy(lens).cuda()))
    check(got, oracle_all(q, k, v, W, Gs, Es, lens))
    # [B, L, H, d] physical layout through strides
    E = random_residual(L, W, 4, seed=8)
    plan = mg.Plan(L, 2, D, W, G, E)
    Qt, Kt, Vt = (x.transpose(1, 2).contiguous().transpose(1, 2) for x in (Q, K, V))
    Ot = torch.empty_like(Qt.transpose(1, 2)).transpose(1, 2)
    check(from_device(mg.sparse_attention_fwd(plan, Qt, Kt, Vt, Ot)), oracle_all(q, k, v, W, G, E))


def test_full_size_c2_d128_sampled():
    c = get_config("C2")
    q, k, v = make_qkv(c.B, c.H, c.L, D, seed=c.seed)
    plan = mg.Plan(c.L, c.H, D, c.window, c.global_idx, c.extra_idx)
    got = from_device(mg.sparse_attention_fwd(plan, *(to_device(x) for x in (q, k, v))))
    assert np.isfinite(got).all()
    rng = np.random.default_rng(17)
    g, ex = global_flags(c.L, c.global_idx), ExtraIndex(c.L, c.extra_idx)
    errs = []
    for (b, h) in [(0, 0), (c.B - 1, c.H - 1), (c.B // 2, 5)]:
        rows = sorted(set(rng.choice(c.L, 48, replace=False).tolist()) | {0, 31, 32, 127, 128, c.L - 1})
        Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
        errs.append(np.abs(got[b, h, rows] - attention_rows(Qh, Kh, Vh, rows, c.window, g, ex)))
    e = np.concatenate(errs)
    assert e.max() <= TOL_MAX and e.mean() <= TOL_MEAN, (e.max(), e.mean())


def test_staged_d128_unsupported():
    plan = mg.Plan(256, 1, D, 32, [0], None)
    Q = torch.zeros(1, 1, 256, D, dtype=torch.bfloat16, device="cuda")
    with pytest.raises(mg.MGError):
        mg.sparse_attention_fwd_staged(plan, Q, Q, Q)
