"""GPU parity of block b = 64 plans, the dilated pattern and the per-pattern autotuned plan
(P:68 dilated, P:111 / P:185 block size 64, P:295-297 blocked patterns).

With b = 64 the coarse part is the b = 64 BSR: its 64-tiles run as quadrants of 128 x 128 tcgen05
tiles with the non-member quadrants masked, and every element outside the 64-tiles is in the
b = 64 CSR residual, so the result is the same masked softmax attention (O-4).
"""
import numpy as np
import pytest
import torch

import paper_conf_iiswc_lica22_b200 as mg
from oracle import ExtraIndex, attention_rows, dense_masked_attention, global_flags, head_inputs_f64
from workloads import blocked_pairs, get_config, make_qkv, random_residual
from gpu_util import TOL_MAX, TOL_MEAN, err_stats, from_device, to_device

pytestmark = pytest.mark.gpu


def oracle_all(q, k, v, window, G, E, lens=None):
    out = np.zeros(q.shape)
    for b in range(q.shape[0]):
        for h in range(q.shape[1]):
            Q, K, V = head_inputs_f64(q, k, v, b, h)
            out[b, h] = dense_masked_attention(Q, K, V, window, G, E, valid_len=None if lens is None else int(lens[b]))
    return out


def check(got, ref):
    mx, mean = err_stats(got, ref)
    assert np.isfinite(got).all()
    assert mx <= TOL_MAX * max(1.0, np.abs(ref).max() / 4) and mean <= TOL_MEAN, (mx, mean)


L, H, B, W = 1024, 3, 2, 128
G = np.array([0, 1, 2, 130, 777], np.int32)


@pytest.mark.parametrize("kw", [{}, dict(strip_max_cols=-1), dict(tau=0.3), dict(num_sms=2), dict(dense_chunk=2)])
def test_block64_mixed_pattern(kw):
    """Band + global rows + random residual + a blocked pattern at b = 64 (the residual and the
    64-tiles not covered by a band go to strips / CSR rows)."""
    E = np.concatenate([random_residual(L, W, 5, seed=3), blocked_pairs(L, 64, lambda I: [(I * 5) % 16])])
    q, k, v = make_qkv(B, H, L, 64, seed=5, dist="adversarial", global_idx=G)
    plan = mg.Plan(L, H, 64, W, G, E, block=64, **kw)
    got = from_device(mg.sparse_attention_fwd(plan, *(to_device(x) for x in (q, k, v))))
    check(got, oracle_all(q, k, v, W, G, E))


@pytest.mark.parametrize("Lr,window,Gr", [(1000, 64, [0, 999]), (300, 40, [5]), (129, 0, []), (192, 512, [])])
def test_block64_ragged(Lr, window, Gr):
    E = np.random.default_rng(Lr).integers(0, Lr, size=(3 * Lr, 2)).astype(np.int32)
    q, k, v = make_qkv(2, 2, Lr, 64, seed=Lr)
    plan = mg.Plan(Lr, 2, 64, window, Gr, E, block=64)
    check(from_device(mg.sparse_attention_fwd(plan, *(to_device(x) for x in (q, k, v)))),
          oracle_all(q, k, v, window, Gr, E))


def test_block64_batched_and_padded():
    Gs = [np.array([0, 5, 700], np.int32), np.array([300], np.int32), np.zeros(0, np.int32),
          np.arange(0, 40, dtype=np.int32)]
    Es = [random_residual(L, W, b + 1, seed=60 + b) for b in range(4)]
    plan = mg.BatchedPlan(L, 2, 64, W, Gs, Es, block=64)
    q, k, v = make_qkv(4, 2, L, 64, seed=52)
    Q, K, V = (to_device(x) for x in (q, k, v))
    lens = np.array([L, 333, 1000, 129], np.int32)
    got = from_device(mg.sparse_attention_fwd_padded(plan, Q, K, V, torch.from_numpy(lens).cuda()))
    for b in range(4):
        for h in range(2):
            Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
            check(got[b, h], dense_masked_attention(Qh, Kh, Vh, W, Gs[b], Es[b], valid_len=int(lens[b])))


def sampled(cfg_name, plan, seed=17):
    c = get_config(cfg_name)
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=c.seed)
    got = from_device(mg.sparse_attention_fwd(plan, *(to_device(x) for x in (q, k, v))))
    assert np.isfinite(got).all()
    rng = np.random.default_rng(seed)
    g, ex = global_flags(c.L, c.global_idx), ExtraIndex(c.L, c.extra_idx)
    errs = []
    for (b, h) in [(0, 0), (c.B - 1, c.H - 1)]:
        rows = sorted(set(rng.choice(c.L, 48, replace=False).tolist()) | {0, 63, 64, 127, c.L - 1})
        Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
        errs.append(np.abs(got[b, h, rows] - attention_rows(Qh, Kh, Vh, rows, c.window, g, ex)))
    e = np.concatenate(errs)
    assert e.max() <= TOL_MAX and e.mean() <= TOL_MEAN, (e.max(), e.mean())


@pytest.mark.parametrize("cfg,b,tau", [("C2", 64, 0.0), ("DIL-LD", 128, 0.0), ("DIL-LD", 64, 0.0),
                                       ("DIL-LD", 64, 0.25), ("F9-RBR", 64, 0.2)])
def test_full_size_block64_and_dilated(cfg, b, tau):
    c = get_config(cfg)
    sampled(cfg, mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx, block=b, tau=tau))


@pytest.mark.parametrize("cfg", ["DIL-LD", "F9-RBR"])
def test_autotuned_plan(cfg):
    """mg_plan_autotune: the candidate plans are timed on the device tensors; the chosen plan's
    forward meets the oracle bar."""
    c = get_config(cfg)
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=c.seed)
    Q, K, V = (to_device(x) for x in (q, k, v))
    plan, chosen, ms = mg.autotune_plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx, Q, K, V)
    assert chosen["block"] in (64, 128) and 0.0 <= chosen["tau"] <= 0.5 and ms > 0
    sampled(cfg, plan)
