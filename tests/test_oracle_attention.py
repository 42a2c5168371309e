"""Pins for the oracle's attention (O-4..O-7) against things other than itself.

* library special case: w >= 2L is dense attention = torch SDPA in fp64 (pins 1/sqrt(d), softmax);
* closed forms: diagonal-only pattern gives O = V; Q = 0 gives the mean of V over the row's mask;
  V = 1 gives O = 1; a global row equals torch.softmax over the full row;
* pure-Python brute force with math.exp on tiny L;
* invariants: row sums of P = 1, P = 0 off the mask, shift invariance, locality (K/V outside the
  mask has no effect);
* cross-checks: CSR reference (O-5) and partitioned LSE reference (O-6) equal O-4 to 1e-12.
"""
import math

import numpy as np
import pytest
import torch

from oracle import (canonical_plan, csr_reference, dense_masked_attention, partitioned_reference,
                    staged_intermediates, union_mask_dense, attention_rows, head_inputs_f64,
                    global_flags, ExtraIndex)
from workloads import get_config, make_qkv, bits_to_f64, random_small_config

E0 = np.zeros((0, 2), np.int32)


def qkv64(L, d=64, seed=0, dist="normal", G=None):
    q, k, v = make_qkv(1, 1, L, d, seed=seed, dist=dist, global_idx=G)
    return head_inputs_f64(q, k, v, 0, 0)


def test_dense_window_equals_torch_sdpa():
    L = 96
    Q, K, V = qkv64(L)
    O = dense_masked_attention(Q, K, V, 2 * L + 2, [], E0)
    ref = torch.nn.functional.scaled_dot_product_attention(
        torch.from_numpy(Q)[None, None], torch.from_numpy(K)[None, None], torch.from_numpy(V)[None, None])
    assert np.abs(O - ref[0, 0].numpy()).max() < 1e-12


def test_diagonal_only_gives_V():
    Q, K, V = qkv64(64)
    O = dense_masked_attention(Q, K, V, 0, [], E0)
    assert np.array_equal(O, V)


def test_zero_q_gives_mask_mean():
    L = 80
    G = np.array([3, 40])
    E = np.array([[0, 70], [5, 60], [5, 61]])
    Q, K, V = qkv64(L, dist="zeros_q")
    O = dense_masked_attention(Q, K, V, 10, G, E)
    M = union_mask_dense(L, 10, G, E)
    for r in range(L):
        assert np.allclose(O[r], V[M[r]].mean(axis=0), atol=1e-13, rtol=0)


def test_ones_v_gives_one():
    Q, K, V = qkv64(100, dist="ones_v")
    O = dense_masked_attention(Q, K, V, 16, [0, 50], np.array([[1, 99]]))
    assert np.abs(O - 1.0).max() < 1e-13


def test_global_row_is_dense_softmax_row():
    L = 128
    G = np.array([7, 100])
    Q, K, V = qkv64(L, seed=4)
    O = dense_masked_attention(Q, K, V, 8, G, E0)
    for r in G:
        s = torch.from_numpy(Q[r] @ K.T / 8.0)
        ref = torch.softmax(s, dim=0).numpy() @ V
        assert np.abs(O[r] - ref).max() < 1e-12


def brute_attention(Q, K, V, M):
    L, d = Q.shape
    out = [[0.0] * V.shape[1] for _ in range(L)]
    for r in range(L):
        cols = [c for c in range(L) if M[r][c]]
        if not cols:
            continue
        s = [sum(Q[r][i] * K[c][i] for i in range(d)) / math.sqrt(d) for c in cols]
        m = max(s)
        e = [math.exp(x - m) for x in s]
        z = sum(e)
        for j in range(V.shape[1]):
            out[r][j] = sum(e[k] * V[cols[k]][j] for k in range(len(cols))) / z
    return np.array(out)


@pytest.mark.parametrize("seed", range(8))
def test_brute_force_tiny(seed):
    rng = np.random.default_rng(seed)
    L, window, G, E = random_small_config(rng, 16)
    Q, K, V = (rng.standard_normal((L, 8)) for _ in range(3))
    M = union_mask_dense(L, window, G, E)
    O = dense_masked_attention(Q, K, V, window, G, E)
    assert np.abs(O - brute_attention(Q, K, V, M)).max() < 1e-12


def test_P_rows_sum_to_one_and_zero_off_mask():
    c = get_config("C1")
    Q, K, V = qkv64(c.L)
    O, P = dense_masked_attention(Q, K, V, c.window, c.global_idx, c.extra_idx, return_P=True)
    M = union_mask_dense(c.L, c.window, c.global_idx, c.extra_idx)
    assert np.abs(P.sum(axis=1) - 1).max() < 1e-12
    assert (P[~M] == 0).all()


def test_shift_invariance():
    L = 64
    Q, K, V = qkv64(L, seed=2)
    u = np.random.default_rng(9).standard_normal(64)
    O1 = dense_masked_attention(Q, K, V, 12, [1], np.array([[3, 50]]))
    O2 = dense_masked_attention(Q, K + u, V, 12, [1], np.array([[3, 50]]))   # S(r, :) += const_r
    assert np.abs(O1 - O2).max() < 1e-10


def test_locality_outside_mask():
    L = 96
    Q, K, V = qkv64(L, seed=3)
    G = np.array([0])
    M = union_mask_dense(L, 8, G, E0)
    O1 = dense_masked_attention(Q, K, V, 8, G, E0)
    K2, V2 = K.copy(), V.copy()
    K2[60] += 5.0
    V2[60] -= 3.0
    O2 = dense_masked_attention(Q, K2, V2, 8, G, E0)
    unaffected = ~M[:, 60]
    assert np.array_equal(O1[unaffected], O2[unaffected])
    assert np.abs(O1[~unaffected] - O2[~unaffected]).max() > 1e-3


@pytest.mark.parametrize("cfg", ["C1"])
def test_csr_and_partitioned_equal_dense(cfg):
    c = get_config(cfg)
    Q, K, V = qkv64(c.L, seed=11, dist="adversarial", G=c.global_idx)
    O = dense_masked_attention(Q, K, V, c.window, c.global_idx, c.extra_idx)
    O5 = csr_reference(Q, K, V, c.window, c.global_idx, c.extra_idx)
    assert np.abs(O5 - O).max() <= 1e-12 * max(1.0, np.abs(O).max())
    for b in (64, 128):
        plan = canonical_plan(c.L, c.window, c.global_idx, c.extra_idx, b)
        O6 = partitioned_reference(Q, K, V, plan)
        assert np.abs(O6 - O).max() <= 1e-12 * max(1.0, np.abs(O).max())


@pytest.mark.parametrize("seed", range(6))
def test_partitioned_equal_dense_random(seed):
    rng = np.random.default_rng(50 + seed)
    L, window, G, E = random_small_config(rng, 48)
    Q, K, V = (rng.standard_normal((L, 16)) * 3 for _ in range(3))
    O = dense_masked_attention(Q, K, V, window, G, E)
    for b in (2, 8, 64):
        O6 = partitioned_reference(Q, K, V, canonical_plan(L, window, G, E, b))
        assert np.abs(O6 - O).max() < 1e-12


def test_attention_rows_matches_dense():
    c = get_config("C1")
    Q, K, V = qkv64(c.L, seed=5)
    O = dense_masked_attention(Q, K, V, c.window, c.global_idx, c.extra_idx)
    rows = [0, 1, 100, 200, 511]
    Or = attention_rows(Q, K, V, rows, c.window, global_flags(c.L, c.global_idx), ExtraIndex(c.L, c.extra_idx))
    assert np.abs(Or - O[rows]).max() < 1e-12


def test_staged_intermediates_reassemble_P():
    L, window = 40, 6
    G, E = np.array([2]), np.array([[10, 39], [30, 0]])
    Q, K, V = qkv64(L, seed=6)
    _, P = dense_masked_attention(Q, K, V, window, G, E, return_P=True)
    plan = canonical_plan(L, window, G, E, 8)
    S_t, S_f, P_t, P_f, S_g, P_g = staged_intermediates(Q, K, plan)
    R = np.zeros((L, L))
    b = plan.block
    for I in range(plan.nb):
        for t in range(plan.bsr_row_ptr[I], plan.bsr_row_ptr[I + 1]):
            J = plan.bsr_col[t]
            R[I * b:I * b + b, J * b:J * b + b] += P_t[t][: min(b, L - I * b), : min(b, L - J * b)]
    rows = np.repeat(np.arange(L), np.diff(plan.csr_row_ptr))
    np.add.at(R, (rows, plan.csr_col), P_f)
    R[plan.global_rows] = P_g
    assert np.abs(R - P).max() < 1e-12
    # S at plan positions: masked-off tile positions are -inf; CSR values are the scaled dots
    assert np.allclose(S_f, np.einsum("nd,nd->n", Q[rows], K[plan.csr_col]) / 8.0)


def test_bf16_inputs_exact_upcast():
    q, k, v = make_qkv(1, 1, 8, 64, seed=0)
    x = bits_to_f64(q)
    # every value is exactly representable in bf16: 8 significant bits
    m, e = np.frexp(x[x != 0])
    assert np.all((m * 2**8) == np.round(m * 2**8))


# ---------------------------------------------------------------- padding (valid length, A18)
@pytest.mark.parametrize("seed", range(6))
def test_padding_equals_truncated_problem(seed):
    """Padding to L with n valid tokens = the same pattern on the first n tokens only (a problem of
    length n, computed without any padding), and O = 0 on the padded rows."""
    rng = np.random.default_rng(700 + seed)
    L = int(rng.integers(40, 160))
    n = int(rng.integers(1, L + 1))
    window = 2 * int(rng.integers(0, 20))
    G = np.unique(rng.integers(0, L, size=int(rng.integers(0, 4)))).astype(np.int32)
    E = rng.integers(0, L, size=(int(rng.integers(0, 3 * L)), 2)).astype(np.int32)
    Q, K, V = (rng.standard_normal((L, 64)) for _ in range(3))
    got = dense_masked_attention(Q, K, V, window, G, E, valid_len=n)
    Gn = G[G < n]
    En = E[(E[:, 0] < n) & (E[:, 1] < n)]
    ref = dense_masked_attention(Q[:n], K[:n], V[:n], window, Gn, En)
    np.testing.assert_allclose(got[:n], ref, rtol=0, atol=1e-12)
    assert (got[n:] == 0).all()
    g = global_flags(L, G)
    rows = list(range(0, L, 7))
    np.testing.assert_allclose(attention_rows(Q, K, V, rows, window, g, ExtraIndex(L, E), valid_len=n),
                               got[rows], rtol=0, atol=1e-12)
