"""Compound sparse attention forward in fp64 (oracle, test infrastructure only).

Per head, with Q_h, K_h, V_h of shape L x D_h (§2.2), the sparse attention
runs "SDDMM, scaling and masking, SpSoftmax, and SpMM" (§2.2):

* SDDMM: S = Q K^T, computed only at non-zero positions;
* scaling: S * SF with SF = 1/sqrt(d) (P:54 is garbled as "L_h / m"; DESIGN.md
  reading A1 follows the cited Vaswani et al. [39]);
* masking: invalid elements get -inf;
* SpSoftmax: row-wise safe softmax over the non-zeros: max, sum of exp(x - max),
  normalise (§3.3);
* SpMM: context C = P V.

``dense_masked_attention`` (O-4) is this definition written out over a dense mask.
``csr_reference`` (O-5) evaluates the same definition row by row over a plain CSR
of M. ``partitioned_reference`` (O-6) evaluates each part of the canonical plan
separately — coarse tiles, CSR residual, dense global rows — and merges their
(max, sum, unnormalised context) by log-sum-exp, as the compound SpSoftmax must
("we sweep the non-zero blocks ... Next, we sweep non-zero elements"; global
rows independent). ``staged_intermediates`` (O-7) returns S and P at plan
positions. All arithmetic is float64; an empty row gives O = 0 (reading A10).
"""
from __future__ import annotations

import math

import numpy as np

from workloads import bits_to_f64

from .mask import ExtraIndex, global_flags, mask_rows, mask_row_cols
from .plan import CanonicalPlan


def head_inputs_f64(Qb, Kb, Vb, b: int, h: int, dtype: str = "bf16"):
    """Exact fp64 upcast of one (batch, head) slice of [B, H, L, d] uint16 bit arrays."""
    return (bits_to_f64(Qb[b, h], dtype), bits_to_f64(Kb[b, h], dtype), bits_to_f64(Vb[b, h], dtype))


def _softmax_rows(S: np.ndarray):
    """Safe softmax per row. Rows that are all -inf give P = 0."""
    m = S.max(axis=1, keepdims=True)
    empty = ~np.isfinite(m)
    m = np.where(empty, 0.0, m)
    p = np.exp(S - m)                       # exp(-inf) = 0 off the mask
    l = p.sum(axis=1, keepdims=True)
    P = np.where(l > 0, p / np.where(l > 0, l, 1.0), 0.0)
    return P


def dense_masked_attention(Q, K, V, window: int, global_idx, extra_idx, *, M=None,
                           chunk: int = 256, return_P: bool = False, valid_len: int | None = None):
    """O-4: S = QK^T/sqrt(d); S[~M] = -inf; P = softmax(S); O = P V, for one head (fp64).

    Rows are processed in chunks so that L = 16384 fits in memory. If ``M`` (L x L bool)
    is given it is used instead of the pattern arguments.

    ``valid_len`` = n (padding, "zero-padding ... masked with -inf"; reading A18):
    tokens at positions >= n are padding, so M(r, c) additionally requires r < n and c < n; the
    padded rows have no valid element and get O = 0 (reading A10).
    """
    L, d = Q.shape
    sf = 1.0 / math.sqrt(d)
    O = np.zeros((L, V.shape[1]), dtype=np.float64)
    Pfull = np.zeros((L, L)) if return_P else None
    if M is None:
        g = global_flags(L, global_idx)
        extra = ExtraIndex(L, extra_idx)
    for r0 in range(0, L, chunk):
        r1 = min(L, r0 + chunk)
        Mb = M[r0:r1] if M is not None else mask_rows(r0, r1, L, window, g, extra)
        if valid_len is not None:
            Mb = Mb & (np.arange(r0, r1) < valid_len)[:, None] & (np.arange(L) < valid_len)[None, :]
        S = (Q[r0:r1] @ K.T) * sf
        S = np.where(Mb, S, -np.inf)
        P = _softmax_rows(S)
        O[r0:r1] = P @ V
        if return_P:
            Pfull[r0:r1] = P
    return (O, Pfull) if return_P else O


def csr_reference(Q, K, V, window: int, global_idx, extra_idx):
    """O-5: a plain CSR of the full union M; per row: gather-dot, safe softmax, gather-axpy."""
    L, d = Q.shape
    sf = 1.0 / math.sqrt(d)
    g = global_flags(L, global_idx)
    extra = ExtraIndex(L, extra_idx)
    row_ptr = [0]
    cols = []
    for r in range(L):
        c = mask_row_cols(r, L, window, g, extra)
        cols.append(c)
        row_ptr.append(row_ptr[-1] + c.size)
    col = np.concatenate(cols) if cols else np.zeros(0, np.int64)
    O = np.zeros((L, V.shape[1]))
    for r in range(L):
        c = col[row_ptr[r]:row_ptr[r + 1]]
        if c.size == 0:
            continue
        s = (K[c] @ Q[r]) * sf
        m = s.max()
        p = np.exp(s - m)
        O[r] = (p / p.sum()) @ V[c]
    return O


def attention_rows(Q, K, V, rows, window: int, gflags: np.ndarray, extra: ExtraIndex,
                   valid_len: int | None = None):
    """The same definition evaluated only at the given rows (for sampled full-size parity);
    ``valid_len`` as in dense_masked_attention."""
    L, d = Q.shape
    sf = 1.0 / math.sqrt(d)
    out = np.zeros((len(rows), V.shape[1]))
    for i, r in enumerate(rows):
        if valid_len is not None and r >= valid_len:
            continue
        c = mask_row_cols(int(r), L, window, gflags, extra)
        if valid_len is not None:
            c = c[c < valid_len]
        if c.size == 0:
            continue
        s = (K[c] @ Q[r]) * sf
        p = np.exp(s - s.max())
        out[i] = (p / p.sum()) @ V[c]
    return out


def _part_stats(s: np.ndarray, Vc: np.ndarray):
    """(m, l, O~) of one part of a row: m = max s, l = sum exp(s - m), O~ = sum exp(s - m) V."""
    if s.size == 0 or not np.isfinite(s).any():
        return -np.inf, 0.0, np.zeros(Vc.shape[1])
    m = s.max()
    p = np.exp(s - m)
    return m, p.sum(), p @ Vc


def _lse_merge(parts):
    """Merge per-part (m, l, O~): m = max m_i; l = sum l_i e^{m_i-m}; O = sum O~_i e^{m_i-m} / l."""
    m = max(p[0] for p in parts)
    if not np.isfinite(m):
        return np.zeros_like(parts[0][2])
    l = sum(p[1] * math.exp(p[0] - m) for p in parts if np.isfinite(p[0]))
    acc = sum(p[2] * math.exp(p[0] - m) for p in parts if np.isfinite(p[0]))
    return acc / l


def partitioned_reference(Q, K, V, plan: CanonicalPlan):
    """O-6: evaluate coarse tiles, CSR residual and dense global rows separately, merge by LSE."""
    L, d = Q.shape
    b = plan.block
    sf = 1.0 / math.sqrt(d)
    O = np.zeros((L, V.shape[1]))
    is_global = np.zeros(L, dtype=bool)
    is_global[plan.global_rows] = True
    for I in range(plan.nb):
        r0, r1 = I * b, min(L, I * b + b)
        # coarse part: gather every tile's valid positions row by row
        coarse_cols = [[] for _ in range(r1 - r0)]
        for t in range(plan.bsr_row_ptr[I], plan.bsr_row_ptr[I + 1]):
            J = plan.bsr_col[t]
            bits = plan.tile_bits(t)
            for a in range(r1 - r0):
                cc = np.nonzero(bits[a])[0] + J * b
                coarse_cols[a].append(cc[cc < L])
        for a in range(r1 - r0):
            r = r0 + a
            if is_global[r]:
                continue
            cc = np.concatenate(coarse_cols[a]) if coarse_cols[a] else np.zeros(0, np.int64)
            fc = plan.csr_col[plan.csr_row_ptr[r]:plan.csr_row_ptr[r + 1]].astype(np.int64)
            parts = [_part_stats((K[cc] @ Q[r]) * sf, V[cc]), _part_stats((K[fc] @ Q[r]) * sf, V[fc])]
            O[r] = _lse_merge(parts)
    for r in plan.global_rows:
        s = (K @ Q[r]) * sf
        O[r] = _lse_merge([_part_stats(s, V)])
    return O


def staged_intermediates(Q, K, plan: CanonicalPlan):
    """O-7: S and P at plan positions.

    Returns (S_tiles [nt, b, b] with -inf where bit = 0, S_csr [nnz], P_tiles, P_csr,
    S_global [G, L], P_global [G, L]).
    """
    L, d = Q.shape
    b = plan.block
    sf = 1.0 / math.sqrt(d)
    nt = plan.n_tiles
    S_t = np.full((nt, b, b), -np.inf)
    S_f = np.zeros(plan.csr_col.size)
    Qp = np.zeros((plan.nb * b, d)); Qp[:L] = Q
    Kp = np.zeros((plan.nb * b, d)); Kp[:L] = K
    for I in range(plan.nb):
        for t in range(plan.bsr_row_ptr[I], plan.bsr_row_ptr[I + 1]):
            J = plan.bsr_col[t]
            full = (Qp[I * b:(I + 1) * b] @ Kp[J * b:(J + 1) * b].T) * sf
            S_t[t] = np.where(plan.tile_bits(t), full, -np.inf)
    rows = np.repeat(np.arange(L), np.diff(plan.csr_row_ptr))
    S_f[:] = np.einsum("nd,nd->n", Q[rows], K[plan.csr_col]) * sf
    # row-wise softmax across both formats
    m = np.full(L, -np.inf)
    for I in range(plan.nb):
        for t in range(plan.bsr_row_ptr[I], plan.bsr_row_ptr[I + 1]):
            r1 = min(L, I * b + b) - I * b
            m[I * b:I * b + r1] = np.maximum(m[I * b:I * b + r1], S_t[t, :r1].max(axis=1))
    np.maximum.at(m, rows, S_f)
    mm = np.where(np.isfinite(m), m, 0.0)
    l = np.zeros(L)
    P_t = np.zeros_like(S_t)
    for I in range(plan.nb):
        for t in range(plan.bsr_row_ptr[I], plan.bsr_row_ptr[I + 1]):
            r1 = min(L, I * b + b) - I * b
            e = np.exp(S_t[t, :r1] - mm[I * b:I * b + r1, None])
            P_t[t, :r1] = e
            l[I * b:I * b + r1] += e.sum(axis=1)
    e_f = np.exp(S_f - mm[rows])
    np.add.at(l, rows, e_f)
    for I in range(plan.nb):
        for t in range(plan.bsr_row_ptr[I], plan.bsr_row_ptr[I + 1]):
            r1 = min(L, I * b + b) - I * b
            P_t[t, :r1] /= np.where(l[I * b:I * b + r1, None] > 0, l[I * b:I * b + r1, None], 1.0)
    P_f = e_f / np.where(l[rows] > 0, l[rows], 1.0)
    G = plan.global_rows
    S_g = (Q[G] @ K.T) * sf
    P_g = _softmax_rows(S_g)
    return S_t, S_f, P_t, P_f, S_g, P_g


def useful_flops(nnz_per_head: int, d: int, B: int, H: int) -> int:
    """Useful flops = 4 * nnz * d * B * H (2d for the QK^T dot, 2d for PV per valid element)."""
    return 4 * int(nnz_per_head) * d * B * H
