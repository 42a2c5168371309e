"""GPU parity of the staged (paper-dataflow) forward, step by step, against the oracle's
intermediates (O-7, oracle.staged_intermediates) and the dense fp64 oracle (O-4).

Each step of SURVEY §8(a) is checked on its own through the C ABI:
  mg_staged_sddmm   -> S at plan positions (a-2 tiles, a-3 CSR, a-4 dense rows), -inf layout exact
  mg_staged_softmax -> P at plan positions (a-5 compound SpSoftmax)
  mg_staged_spmm    -> O (a-6 CSR SpMM, a-7 tile SpMM, a-4 dense rows, a-8 merge)
Tolerances: S to 1e-3 * (1 + |S|) (bf16 products are exact in fp32, only the summation order
differs); P and O to the north_star bar (max 2e-2, mean 2e-3).
"""
import numpy as np
import pytest
import torch

import paper_conf_iiswc_lica22_b200 as mg
from oracle import canonical_plan, dense_masked_attention, head_inputs_f64, staged_intermediates
from workloads import get_config, make_qkv, random_residual
from gpu_util import TOL_MAX, TOL_MEAN, err_stats, from_device, to_device

pytestmark = pytest.mark.gpu

CASES = {
    # name: (B, H, L, window, G, E-generator)
    "c1": (1, 1, 512, 64, [0, 200], None),
    "mixed": (2, 2, 1024, 128, [0, 1, 2, 130, 777], lambda L: random_residual(L, 128, 6, seed=3)),
    "ragged": (1, 2, 1000, 64, [0, 999], lambda L: np.random.default_rng(L).integers(0, L, (3 * L, 2)).astype(np.int32)),
    "no_global": (1, 1, 384, 32, [], lambda L: random_residual(L, 32, 4, seed=1)),
}


def _f32(t):
    return t.float().cpu().numpy().astype(np.float64)


def _check_S(got, ref):
    inf_g, inf_r = np.isneginf(got), np.isneginf(ref)
    assert np.array_equal(inf_g, inf_r), "masked (-inf) positions differ"
    fin = ~inf_r
    if fin.any():
        err = np.abs(got[fin] - ref[fin]) / (1.0 + np.abs(ref[fin]))
        assert err.max() <= 1e-3, err.max()


def _check_P(got, ref):
    if ref.size:
        mx, mean = err_stats(got, ref)
        assert mx <= TOL_MAX and mean <= TOL_MEAN, (mx, mean)


@pytest.mark.parametrize("case", sorted(CASES))
@pytest.mark.parametrize("dtype", ["bf16", "fp16"])
def test_staged_steps_match_oracle(case, dtype):
    B, H, L, window, G, egen = CASES[case]
    G = np.array(G, np.int32)
    E = egen(L) if egen else np.zeros((0, 2), np.int32)
    q, k, v = make_qkv(B, H, L, 64, seed=21, dist="adversarial", global_idx=G, dtype=dtype)
    plan = mg.Plan(L, H, 64, window, G, E)
    Q, K, V = (to_device(x, dtype) for x in (q, k, v))
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float16
    bufs = mg.staged_buffers(plan, B, tdt)
    lpad = bufs["lpad"]
    mg.staged_sddmm(plan, Q, K, bufs)
    mg.staged_softmax(plan, B, bufs)
    O = torch.empty_like(Q)
    mg.staged_spmm(plan, V, O, bufs)
    torch.cuda.synchronize()

    cp = canonical_plan(L, window, G, E, block=128)
    nt, nG = cp.n_tiles, len(cp.global_rows)
    St, Sf, Sg = _f32(bufs["S_tiles"]), _f32(bufs["S_csr"]), _f32(bufs["S_global"])
    Pt, Pf, Pg = (from_device(bufs[n]) for n in ("P_tiles", "P_csr", "P_global"))
    Og = from_device(O)
    for b in range(B):
        for h in range(H):
            u = b * H + h
            Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h, dtype)
            S_t, S_f, P_t, P_f, S_g, P_g = staged_intermediates(Qh, Kh, cp)
            _check_S(St[u].reshape(nt, 128, 128), S_t)
            _check_S(Sf[u], S_f)
            sg = Sg[u].reshape(nG, lpad)
            _check_S(sg[:, :L], S_g)
            assert np.isneginf(sg[:, L:]).all()
            _check_P(Pt[u].reshape(nt, 128, 128), P_t)
            _check_P(Pf[u], P_f)
            pg = Pg[u].reshape(nG, lpad)
            _check_P(pg[:, :L], P_g)
            assert (pg[:, L:] == 0).all()
            ref = dense_masked_attention(Qh, Kh, Vh, window, G, E)
            mx, mean = err_stats(Og[b, h], ref)
            assert mx <= TOL_MAX and mean <= TOL_MEAN, (b, h, mx, mean)


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_staged_forward_matches_fused(cfg):
    """mg_sparse_attention_fwd_staged (plan-owned buffers) against the oracle on C1, and against the
    fused forward on C2 at full size (both within the bar of the oracle on sampled rows)."""
    c = get_config(cfg)
    B = c.B if cfg == "C1" else 1
    q, k, v = make_qkv(B, c.H, c.L, c.d, seed=c.seed)
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
    Q, K, V = (to_device(x) for x in (q, k, v))
    Os = from_device(mg.sparse_attention_fwd_staged(plan, Q, K, V))
    Of = from_device(mg.sparse_attention_fwd(plan, Q, K, V))
    torch.cuda.synchronize()
    if cfg == "C1":
        Qh, Kh, Vh = head_inputs_f64(q, k, v, 0, 0)
        ref = dense_masked_attention(Qh, Kh, Vh, c.window, c.global_idx, c.extra_idx)
        mx, mean = err_stats(Os[0, 0], ref)
        assert mx <= TOL_MAX and mean <= TOL_MEAN
    mx, mean = err_stats(Os, Of)
    assert mx <= TOL_MAX and mean <= TOL_MEAN, (mx, mean)


def test_staged_rejects_null_buffers():
    c = get_config("C1")
    plan = mg.Plan(c.L, 1, 64, c.window, c.global_idx, c.extra_idx)
    Q = torch.zeros(1, 1, c.L, 64, dtype=torch.bfloat16, device="cuda")
    bufs = mg.staged_buffers(plan, 1, torch.bfloat16)
    bufs["S_tiles"] = None
    with pytest.raises(mg.MGError):
        mg.staged_sddmm(plan, Q, Q, bufs)


@pytest.mark.parametrize("kw", [dict(strip_max_cols=-1), {}, dict(force_all_fine=True)])
def test_staged_multi_stream_bit_identical(kw):
    """MG_STAGED_MULTI_STREAM (coarse || fine kernels of each step on two streams):
    bit-identical to the single-stream staged forward and within the bar of the oracle; repeated
    calls reuse the plan's side stream and event."""
    L, H, B, w = 1024, 2, 2, 128
    G = np.array([0, 3, 600], np.int32)
    E = random_residual(L, w, 5, seed=8)
    q, k, v = make_qkv(B, H, L, 64, seed=19, dist="adversarial", global_idx=G)
    plan = mg.Plan(L, H, 64, w, G, E, **kw)
    Q, K, V = (to_device(x) for x in (q, k, v))
    one = from_device(mg.sparse_attention_fwd_staged(plan, Q, K, V))
    for _ in range(3):
        two = from_device(mg.sparse_attention_fwd_staged(plan, Q, K, V, multi_stream=True))
        assert np.array_equal(one, two)
    for b in range(B):
        for h in range(H):
            Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
            ref = dense_masked_attention(Qh, Kh, Vh, w, G, E)
            mx, mean = err_stats(two[b, h], ref)
            assert mx <= TOL_MAX * max(1.0, np.abs(ref).max() / 4) and mean <= TOL_MEAN, (b, h, mx, mean)
