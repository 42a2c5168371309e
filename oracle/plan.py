"""Canonical Multigrain partition of the union mask (oracle, test infrastructure only).

Multigrain "classif[ies] and group[s] sparse patterns into coarse-grained and
fine-grained patterns" and "generate[s] the metadata (e.g., row offsets and column
indices) ... before inferring the model" (§3.1 steps 1-2). Local patterns go to
the coarse BSR kernel, selected/random to the fine CSR kernel (§3.1), global
rows are processed densely and independently (§3.1; §3.3), and
overlapped elements are invalidated so nothing is counted twice (§3.3).

Integer-exact rules (readings A4-A7), block b:

* global_rows = sorted unique G.
* T = {(I, J) : exists r in [Ib, Ib+b) \\ G, c in [Jb, Jb+b), |r-c| <= w/2}
  (every tile touched by the band of a non-global row is coarse; tau = 0), or, with a density
  threshold tau > 0 (reading A17: "sparse blocks with low sparsity"
  favour the fine kernel, dense blocks the coarse one),
  T = {(I, J) : #{(r, c) in tile : M(r, c), r not in G} >= tau * b * b}.
* BSR: bsr_row_ptr[nb+1], bsr_col[] ascending J within each row block.
* tile mask bit (a, beta) = M(Ib+a, Jb+beta) AND NOT G[Ib+a], zero outside [0, L);
  row-major, ceil(b/64) uint64 words per tile row, LSB = lowest column.
* CSR: for r not in G, ascending c with M(r, c) AND (r//b, c//b) not in T. Empty for r in G.

Invariant: popcount(tile masks) + nnz(CSR) + |G| * L = |M|, parts pairwise disjoint.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .mask import ExtraIndex, global_flags, mask_rows


def _words_per_row(b: int) -> int:
    """uint64 words per tile row: ceil(b / 64)."""
    return -(-b // 64)


@dataclass
class CanonicalPlan:
    L: int
    window: int
    block: int
    global_rows: np.ndarray   # int32 [G]
    bsr_row_ptr: np.ndarray   # int32 [nb+1]
    bsr_col: np.ndarray       # int32 [nt]
    tile_masks: np.ndarray    # uint64 [nt, b, ceil(b/64)]
    csr_row_ptr: np.ndarray   # int32 [L+1]
    csr_col: np.ndarray       # int32 [nnz]

    @property
    def nb(self) -> int:
        return -(-self.L // self.block)

    @property
    def n_tiles(self) -> int:
        return int(self.bsr_col.size)

    def tile_bits(self, t: int) -> np.ndarray:
        """Boolean b x b bits of tile t (unpacked from the uint64 words)."""
        b = self.block
        wpr = _words_per_row(b)
        by = self.tile_masks[t].reshape(b, wpr).copy().view(np.uint8).reshape(b, wpr * 8)
        return np.unpackbits(by, axis=1, bitorder="little").astype(bool)[:, :b]

    def tile_popcount(self) -> np.ndarray:
        if self.n_tiles == 0:
            return np.zeros(0, dtype=np.int64)
        by = self.tile_masks.reshape(self.n_tiles, -1).view(np.uint8)
        return np.unpackbits(by, axis=1).sum(axis=1)

    def n_full_tiles(self) -> int:
        return int((self.tile_popcount() == self.block * self.block).sum())


def canonical_plan(L: int, window: int, global_idx, extra_idx, block: int = 128,
                   tau: float = 0.0) -> CanonicalPlan:
    if block < 1 or (block > 64 and block % 64):
        raise ValueError("block must be <= 64 or a multiple of 64")
    if not 0.0 <= tau <= 1.0:
        raise ValueError("tau must be in [0, 1]")
    b = block
    wpr = _words_per_row(b)
    w1 = window // 2
    nb = -(-L // b)
    g = global_flags(L, global_idx)
    extra = ExtraIndex(L, extra_idx)
    global_rows = np.nonzero(g)[0].astype(np.int32)

    row_ptr = [0]
    cols, masks = [], []
    csr_row_ptr = np.zeros(L + 1, dtype=np.int64)
    csr_cols = []
    for I in range(nb):
        r0, r1 = I * b, min(I * b + b, L)
        M = mask_rows(r0, r1, L, window, g, extra)          # (r1-r0) x L
        Mc = M & ~g[r0:r1, None]                            # global rows leave tiles and CSR
        in_T = np.zeros(nb, dtype=bool)
        if tau == 0.0:
            # Tile set of this row block: band of every non-global row.
            for r in range(r0, r1):
                if g[r]:
                    continue
                in_T[max(0, r - w1) // b: min(L - 1, r + w1) // b + 1] = True
        else:
            # Tile set by density: union elements of non-global rows in the tile >= tau * b^2.
            for J in range(nb):
                in_T[J] = Mc[:, J * b: min(J * b + b, L)].sum() >= tau * b * b
        Js = np.nonzero(in_T)[0]
        for J in Js:
            c0, c1 = J * b, min(J * b + b, L)
            bits = np.zeros((b, wpr * 64), dtype=bool)
            bits[: r1 - r0, : c1 - c0] = Mc[:, c0:c1]
            words = np.packbits(bits, axis=1, bitorder="little").view(np.uint64)
            masks.append(words.reshape(b, wpr))
            cols.append(J)
        row_ptr.append(len(cols))
        # CSR residual: union elements whose tile is not coarse.
        col_in_T = np.repeat(in_T, b)[:L]
        R = Mc & ~col_in_T[None, :]
        for i in range(r1 - r0):
            cc = np.nonzero(R[i])[0]
            csr_cols.append(cc)
            csr_row_ptr[r0 + i + 1] = cc.size
    csr_row_ptr = np.cumsum(csr_row_ptr)
    if csr_row_ptr[-1] >= 2**31:
        raise OverflowError("CSR nnz exceeds int32")
    csr_col = np.concatenate(csr_cols).astype(np.int32) if csr_cols else np.zeros(0, np.int32)
    tile_masks = (np.stack(masks) if masks else np.zeros((0, b, wpr), np.uint64)).astype(np.uint64)
    return CanonicalPlan(
        L=L, window=window, block=b, global_rows=global_rows,
        bsr_row_ptr=np.asarray(row_ptr, dtype=np.int32), bsr_col=np.asarray(cols, dtype=np.int32),
        tile_masks=tile_masks, csr_row_ptr=csr_row_ptr.astype(np.int32), csr_col=csr_col,
    )
