"""Seeded synthetic workload generators shared by the oracle tests, the GPU parity tests and bench.py.

This module draws inputs only. It holds none of Multigrain's arithmetic: no mask
union, no tile classification, no softmax. Both sides receive exactly the
arrays produced here.

* Q/K/V recipe: ``numpy.random.default_rng(seed + i)`` (PCG64)
  draws Q (i=0), K (i=1), V (i=2) as float32 standard normals. They are rounded
  to bf16 (or fp16) with round-to-nearest-even and returned as uint16 bit
  patterns. The GPU receives these bits; the oracle upcasts them exactly to fp64.
* Pattern recipe (BASELINE.json ``configs``):
  - C1: B=1, H=1, L=512, w=64, G={0, 200}, E=∅;
  - C2: Longformer-base, B=8, H=12, L=4096, w=512, G=[0,32), E=∅;
  - C3: QDS, B=8, H=12, L=2048, w=256, G=[0,8) ∪ 56 sentence starts drawn by
    ``default_rng(1).choice(arange(8, 2048), 56, replace=False)``, E=∅;
  - C4: Longformer-large long doc, B=2, H=16, L=16384, w=512, G=∅,
    E = 164 (=⌈0.01·L⌉) distinct uniform columns per row outside the band,
    drawn row by row from ``default_rng(0)``;
  - C5: C2's shape at B=64 (sharded over ranks in the scaling bench).
* Paper-faithful extra workloads (reading A15):
  - QDS-LS: QDS-Transformer as local + selected: B=8, H=12, L=2048, w=128 (the window
    whose 64-blocks give P:185's 2:1 sparse:dense ratio), the C3 special tokens as column-only
    selected tokens (every row attends to them, "all-to-one"), no global rows;
  - Fig. 9 synthetic compound patterns (batch 1, L=4096, 4 heads, d=64, 95% sparsity
    per row, i.e. ~205 non-zeros per row): F9-LS (local w=128 + 76 selected columns), F9-LSG
    (local w=128 + 64 selected columns + 12 global tokens), F9-LBR (blocked local, 64-blocks,
    + 141 random columns per row), F9-RBR (blocked random: each 64-row block attends to two
    random 64-column blocks, + 77 random columns per row). Selected columns, random columns and
    block choices are drawn from ``default_rng(seed)`` in a fixed order (see the builders).
  Paper context: local/global/selected/random atomic patterns, PAPER.md
  lines 64-71 (§2.3); Longformer = L+S+G, QDS = L+S.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

__all__ = [
    "Config", "CONFIGS", "get_config", "make_qkv", "to_bf16_bits", "to_fp16_bits",
    "bits_to_f64", "random_residual", "qds_globals", "random_small_config", "selected_columns",
    "blocked_pairs", "uniform_random_pairs", "EXTRA_WORKLOADS",
]


def to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """float32 -> bf16 bit pattern (uint16), round-to-nearest-even; NaN kept quiet."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    u = x.view(np.uint32).astype(np.uint64)
    rounding = ((u >> 16) & 1) + 0x7FFF
    r = ((u + rounding) >> 16).astype(np.uint16)
    nan = np.isnan(x)
    if nan.any():
        r[nan] = 0x7FC0
    return r


def to_fp16_bits(x: np.ndarray) -> np.ndarray:
    """float32 -> IEEE fp16 bit pattern (uint16), numpy's round-to-nearest-even."""
    return np.ascontiguousarray(x, dtype=np.float32).astype(np.float16).view(np.uint16)


def bits_to_f64(bits: np.ndarray, dtype: str = "bf16") -> np.ndarray:
    """Exact upcast of 16-bit patterns to float64."""
    bits = np.asarray(bits, dtype=np.uint16)
    if dtype == "bf16":
        return (bits.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    if dtype == "fp16":
        return bits.view(np.float16).astype(np.float64)
    raise ValueError(dtype)


@dataclass(frozen=True)
class Config:
    name: str
    B: int
    H: int
    L: int
    d: int
    window: int
    global_idx: np.ndarray = field(compare=False)
    extra_idx: np.ndarray = field(compare=False)   # int32 [n, 2] COO (row, col)
    seed: int = 0
    note: str = ""

    @property
    def w1(self) -> int:
        return self.window // 2


def qds_globals(L: int = 2048, n_prefix: int = 8, n_sent: int = 56, seed: int = 1) -> np.ndarray:
    """QDS-style sentence-level global tokens: [0, n_prefix) ∪ n_sent sorted irregular positions."""
    rng = np.random.default_rng(seed)
    sent = np.sort(rng.choice(np.arange(n_prefix, L), n_sent, replace=False))
    return np.concatenate([np.arange(n_prefix), sent]).astype(np.int32)


def random_residual(L: int, window: int, per_row: int, seed: int = 0) -> np.ndarray:
    """Random fine-grained residual: per row r, `per_row` distinct uniform columns
    with |r-c| > window/2, drawn in row order from default_rng(seed). Returns int32 [L*per_row, 2]."""
    w1 = window // 2
    rng = np.random.default_rng(seed)
    cols = np.arange(L)
    out = np.empty((L * per_row, 2), dtype=np.int32)
    for r in range(L):
        cand = cols[np.abs(cols - r) > w1]
        k = min(per_row, cand.size)
        pick = rng.choice(cand, k, replace=False) if k else np.empty(0, np.int64)
        out[r * per_row:r * per_row + k, 0] = r
        out[r * per_row:r * per_row + k, 1] = pick
    return out


_EMPTY_E = np.zeros((0, 2), dtype=np.int32)


def selected_columns(L: int, cols: np.ndarray) -> np.ndarray:
    """Column-only "selected" tokens (all-to-one): every row r attends to every c in cols."""
    cols = np.asarray(cols, dtype=np.int32)
    r = np.repeat(np.arange(L, dtype=np.int32), cols.size)
    return np.stack([r, np.tile(cols, L)], axis=1).astype(np.int32)


def blocked_pairs(L: int, block: int, col_blocks_of_row_block) -> np.ndarray:
    """Blocked pattern: row block I attends all-to-all to each column block in
    col_blocks_of_row_block(I)."""
    out = []
    nb = (L + block - 1) // block
    for I in range(nb):
        rows = np.arange(I * block, min(L, I * block + block), dtype=np.int32)
        for J in col_blocks_of_row_block(I):
            cols = np.arange(J * block, min(L, J * block + block), dtype=np.int32)
            out.append(np.stack([np.repeat(rows, cols.size), np.tile(cols, rows.size)], axis=1))
    return np.concatenate(out).astype(np.int32) if out else _EMPTY_E


def uniform_random_pairs(L: int, per_row: int, seed: int) -> np.ndarray:
    """Per row `per_row` distinct uniform columns over [0, L), drawn row by row (random pattern)."""
    rng = np.random.default_rng(seed)
    out = np.empty((L * per_row, 2), dtype=np.int32)
    for r in range(L):
        out[r * per_row:(r + 1) * per_row, 0] = r
        out[r * per_row:(r + 1) * per_row, 1] = rng.choice(L, per_row, replace=False)
    return out


def dilated_pairs(L: int, stride: int, taps: int) -> np.ndarray:
    """Dilated pattern ("tokens located at a constant stride distance", used "as a dilated
    local pattern combined with a local pattern"): every row r attends to r + k * stride for
    k = +-1 .. +-taps (inside [0, L)). Entries that fall inside a local window are absorbed by the
    plan's set semantics. Returns int32 [n, 2] (row, col) pairs."""
    r = np.arange(L, dtype=np.int64)
    out = []
    for k in range(1, taps + 1):
        for sgn in (1, -1):
            c = r + sgn * k * stride
            ok = (c >= 0) & (c < L)
            out.append(np.stack([r[ok], c[ok]], axis=1))
    return np.concatenate(out).astype(np.int32) if out else np.zeros((0, 2), np.int32)


def _dil() -> "Config":
    L = 4096
    return Config("DIL-LD", 1, 4, L, 64, 256, np.zeros(0, np.int32), dilated_pairs(L, 16, 32), 0,
                  "local w=256 + dilated local (stride 16, 32 taps each side, P:68)")


def _f9(name: str) -> "Config":
    L, rng = 4096, np.random.default_rng(9)
    if name == "F9-LS":
        sel = np.sort(rng.choice(L, 76, replace=False))
        return Config(name, 1, 4, L, 64, 128, np.zeros(0, np.int32), selected_columns(L, sel), 0,
                      "Fig. 9 L+S: local w=128 + 76 selected columns, 95% sparsity per row")
    if name == "F9-LSG":
        sel = np.sort(rng.choice(L, 76, replace=False))
        return Config(name, 1, 4, L, 64, 128, sel[:12].astype(np.int32), selected_columns(L, sel[12:]), 0,
                      "Fig. 9 L+S+G: local w=128 + 64 selected columns + 12 global tokens")
    if name == "F9-LBR":
        E = np.concatenate([blocked_pairs(L, 64, lambda I: [I]), uniform_random_pairs(L, 141, seed=10)])
        return Config(name, 1, 4, L, 64, 0, np.zeros(0, np.int32), E, 0,
                      "Fig. 9 LB+R: blocked local (64-blocks) + 141 random columns per row")
    if name == "F9-RBR":
        nb = L // 64
        picks = [np.sort(rng.choice(nb, 2, replace=False)) for _ in range(nb)]
        E = np.concatenate([blocked_pairs(L, 64, lambda I: picks[I]), uniform_random_pairs(L, 77, seed=11)])
        return Config(name, 1, 4, L, 64, 0, np.zeros(0, np.int32), E, 0,
                      "Fig. 9 RB+R: two random 64-column blocks per 64-row block + 77 random columns")
    raise KeyError(name)


def _qds_ls() -> "Config":
    L = 2048
    return Config("QDS-LS", 8, 12, L, 64, 128, np.zeros(0, np.int32), selected_columns(L, qds_globals(L)), 0,
                  "QDS-Transformer as L+S: w=128, 64 special tokens as column-only selected tokens, B=8")


EXTRA_WORKLOADS = ("QDS-LS", "F9-LS", "F9-LSG", "F9-LBR", "F9-RBR", "DIL-LD")


def _build_configs():
    c = {}
    c["C1"] = Config("C1", 1, 1, 512, 64, 64, np.array([0, 200], np.int32), _EMPTY_E, 0,
                     "single head, L=512, window 64 + 2 global tokens")
    c["C2"] = Config("C2", 8, 12, 4096, 64, 512, np.arange(32, dtype=np.int32), _EMPTY_E, 0,
                     "Longformer-base L=4096, w=512, G=[0,32), B=8")
    c["C3"] = Config("C3", 8, 12, 2048, 64, 256, qds_globals(), _EMPTY_E, 0,
                     "QDS L=2048, w=256, 64 irregular global tokens, B=8")
    c["C5"] = Config("C5", 64, 12, 4096, 64, 512, np.arange(32, dtype=np.int32), _EMPTY_E, 0,
                     "C2 shape at B=64 (scaling sweep)")
    return c


CONFIGS = _build_configs()
_C4_CACHE: dict = {}


def get_config(name: str) -> Config:
    """Return a BASELINE config by name (C1..C5) or a paper-faithful extra workload (EXTRA_WORKLOADS).
    C4's residual is generated on first use (~1 s)."""
    if name in EXTRA_WORKLOADS:
        if name not in _C4_CACHE:
            _C4_CACHE[name] = _qds_ls() if name == "QDS-LS" else (_dil() if name == "DIL-LD" else _f9(name))
        return _C4_CACHE[name]
    if name == "C4":
        if "C4" not in _C4_CACHE:
            L = 16384
            _C4_CACHE["C4"] = Config("C4", 2, 16, L, 64, 512, np.zeros(0, np.int32),
                                     random_residual(L, 512, math.ceil(0.01 * L), seed=0), 0,
                                     "Longformer-large L=16384, w=512, 1% random residual, B=2")
        return _C4_CACHE["C4"]
    return CONFIGS[name]


def make_qkv(B: int, H: int, L: int, d: int, seed: int = 0, dist: str = "normal",
             global_idx: np.ndarray | None = None, dtype: str = "bf16"):
    """Q, K, V as uint16 bit patterns of shape [B, H, L, d].

    dist: "normal" (N(0,1)), "peaky" (Q x 4), "adversarial" (K rows at global positions x 8),
    "zeros_q" (Q = 0), "ones_v" (V = 1).
    """
    shape = (B, H, L, d)
    q = np.random.default_rng(seed + 0).standard_normal(shape, dtype=np.float32)
    k = np.random.default_rng(seed + 1).standard_normal(shape, dtype=np.float32)
    v = np.random.default_rng(seed + 2).standard_normal(shape, dtype=np.float32)
    if dist == "peaky":
        q *= 4.0
    elif dist == "adversarial":
        if global_idx is not None and len(global_idx):
            k[:, :, np.asarray(global_idx), :] *= 8.0
    elif dist == "zeros_q":
        q[...] = 0.0
    elif dist == "ones_v":
        v[...] = 1.0
    elif dist != "normal":
        raise ValueError(dist)
    conv = to_bf16_bits if dtype == "bf16" else to_fp16_bits
    return conv(q), conv(k), conv(v)


def random_small_config(rng: np.random.Generator, L_max: int = 64):
    """A random tiny pattern for brute-force tests: (L, window, G, E)."""
    L = int(rng.integers(1, L_max + 1))
    window = 2 * int(rng.integers(0, L + 2))
    nG = int(rng.integers(0, min(L, 4) + 1))
    G = rng.choice(L, nG, replace=False).astype(np.int32) if nG else np.zeros(0, np.int32)
    nE = int(rng.integers(0, 2 * L + 1))
    E = rng.integers(0, L, size=(nE, 2)).astype(np.int32)
    return L, window, G, E
