"""Union mask M of a compound sparse pattern (oracle, test infrastructure only).

Definition (readings A2/A3):

    M(r, c) = |r - c| <= w/2  OR  G[r]  OR  G[c]  OR  (r, c) in E

* local pattern: "attends the window-sized tokens on both sides with the current
  token" (§2.3), read as |r-c| <= window/2 (reading A2);
* global / selected: "attends the current token to all tokens with a one-to-all
  or all-to-one fashion" (§2.3); a global token is both (reading A3);
* random / arbitrary residual: "the current token attends to the random token"
  (§2.3), given as COO pairs E, with set semantics (duplicates collapse).
"""
from __future__ import annotations

import numpy as np


def global_flags(L: int, global_idx) -> np.ndarray:
    g = np.zeros(L, dtype=bool)
    gi = np.asarray(global_idx, dtype=np.int64).reshape(-1)
    if gi.size:
        g[gi] = True
    return g


class ExtraIndex:
    """Set of extra (row, col) pairs, grouped by row: sorted unique columns per row."""

    def __init__(self, L: int, extra_idx):
        e = np.asarray(extra_idx, dtype=np.int64).reshape(-1, 2)
        if e.size:
            key = np.unique(e[:, 0] * L + e[:, 1])
            rows, cols = key // L, key % L
        else:
            rows = cols = np.zeros(0, dtype=np.int64)
        self.L = L
        self.row_ptr = np.zeros(L + 1, dtype=np.int64)
        np.add.at(self.row_ptr, rows + 1, 1)
        self.row_ptr = np.cumsum(self.row_ptr)
        self.cols = cols

    def row(self, r: int) -> np.ndarray:
        return self.cols[self.row_ptr[r]:self.row_ptr[r + 1]]


def union_mask_dense(L: int, window: int, global_idx, extra_idx) -> np.ndarray:
    """The full L x L boolean union mask (small L only)."""
    w1 = window // 2
    r = np.arange(L)[:, None]
    c = np.arange(L)[None, :]
    M = np.abs(r - c) <= w1
    g = global_flags(L, global_idx)
    M |= g[:, None]
    M |= g[None, :]
    e = np.asarray(extra_idx, dtype=np.int64).reshape(-1, 2)
    if e.size:
        M[e[:, 0], e[:, 1]] = True
    return M


def mask_rows(r0: int, r1: int, L: int, window: int, gflags: np.ndarray, extra: ExtraIndex) -> np.ndarray:
    """Rows [r0, r1) of M as a dense (r1-r0) x L boolean block."""
    w1 = window // 2
    r = np.arange(r0, r1)[:, None]
    c = np.arange(L)[None, :]
    M = np.abs(r - c) <= w1
    M |= gflags[r0:r1, None]
    M |= gflags[None, :]
    for i, rr in enumerate(range(r0, r1)):
        cols = extra.row(rr)
        if cols.size:
            M[i, cols] = True
    return M


def mask_row_cols(r: int, L: int, window: int, gflags: np.ndarray, extra: ExtraIndex) -> np.ndarray:
    """Ascending column indices c with M(r, c)."""
    if gflags[r]:
        return np.arange(L)
    w1 = window // 2
    band = np.arange(max(0, r - w1), min(L - 1, r + w1) + 1)
    return np.union1d(np.union1d(band, np.nonzero(gflags)[0]), extra.row(r))
