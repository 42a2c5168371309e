"""Pins for the oracle's mask (O-2) and canonical plan (O-3) against things other than itself.

* closed-form element and tile counts (SURVEY.md §8(c) "Pins", derived by counting);
* the paper's own block ratios at b=64 (§5.1): Longformer 1:3 sparse:dense,
  QDS 2:1 — these pin the window reading A2 (|r-c| <= w/2);
* a hand-worked example (tests/golden/worked_example_L8.json);
* an element-by-element brute-force re-derivation on tiny random patterns;
* invariants: disjointness, union count, global rows cleared, set semantics.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import canonical_plan, union_mask_dense
from workloads import get_config, random_small_config

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
E0 = np.zeros((0, 2), np.int32)


# ---------------------------------------------------------------- closed forms
def band_nnz(L, w1):
    return L * (2 * w1 + 1) - w1 * (w1 + 1)


def contiguous_global_extra(L, w1, g):
    # globals [0, g), g <= w1 + 1: each global row/col adds its off-band part, minus the g x g overlap
    return 2 * (g * L - g * (w1 + 1) - g * (g - 1) // 2)


def band_tiles(nb, b, w1):
    k = -(-w1 // b)
    return nb * (2 * k + 1) - k * (k + 1)


def full_tiles(nb, b, w1):
    kf = (w1 - b + 1) // b
    return max(0, nb * (2 * kf + 1) - kf * (kf + 1))


@pytest.mark.parametrize("L,window", [(512, 64), (1024, 2), (2048, 256), (4096, 512), (600, 100), (64, 0)])
def test_band_count_closed_form(L, window):
    M = union_mask_dense(L, window, [], E0)
    assert M.sum() == band_nnz(L, window // 2)


@pytest.mark.parametrize("L,window,g", [(4096, 512, 32), (512, 64, 2), (1000, 40, 21), (300, 10, 6)])
def test_contiguous_globals_closed_form(L, window, g):
    w1 = window // 2
    assert g <= w1 + 1
    M = union_mask_dense(L, window, np.arange(g), E0)
    assert M.sum() == band_nnz(L, w1) + contiguous_global_extra(L, w1, g)


def test_config_nnz_values():
    # SURVEY.md §8(c) pins: C2 = 2,280,160 (band 2,035,456); C1 = 34,074.
    assert band_nnz(4096, 256) == 2_035_456
    assert band_nnz(4096, 256) + contiguous_global_extra(4096, 256, 32) == 2_280_160
    c1 = get_config("C1")
    assert union_mask_dense(c1.L, c1.window, c1.global_idx, c1.extra_idx).sum() == 34_074


@pytest.mark.parametrize("L,window,b", [(4096, 512, 64), (4096, 512, 128), (2048, 256, 64), (2048, 256, 128),
                                        (16384, 512, 128), (1024, 100, 64), (512, 0, 64)])
def test_tile_counts_closed_form(L, window, b):
    assert L % b == 0
    nb, w1 = L // b, window // 2
    p = canonical_plan(L, window, [], E0, b)
    assert p.n_tiles == band_tiles(nb, b, w1)
    assert p.n_full_tiles() == full_tiles(nb, b, w1)


def test_paper_block_ratios_P185():
    """'the ratios between the number of the sparse blocks and dense blocks are 1:3 and 2:1,
    respectively, when performing the sparse operation of a local pattern with a block size of 64 in
    Longformer and QDS-Transformer'. Under reading A2 (|r-c| <= w/2):
    Longformer w=512, L=4096 -> 120 partial : 436 full (1:3.6; the one-sided reading gives 1:8);
    QDS w=128, L=2048 -> 62 partial : 32 full (1.94:1)."""
    lf = canonical_plan(4096, 512, [], E0, 64)
    lf_full = lf.n_full_tiles()
    lf_partial = lf.n_tiles - lf_full
    assert (lf_partial, lf_full) == (120, 436)
    assert 2.5 <= lf_full / lf_partial < 4.5          # "1:3"
    qds = canonical_plan(2048, 128, [], E0, 64)
    q_full = qds.n_full_tiles()
    q_partial = qds.n_tiles - q_full
    assert (q_partial, q_full) == (62, 32)
    assert 1.5 <= q_partial / q_full < 2.5            # "2:1"


# ---------------------------------------------------------------- golden example
def test_worked_example_L8():
    g = json.load(open(os.path.join(GOLDEN, "worked_example_L8.json")))
    M = union_mask_dense(g["L"], g["window"], g["global_idx"], np.asarray(g["extra_idx"]).reshape(-1, 2))
    assert [list(np.nonzero(M[r])[0]) for r in range(g["L"])] == g["mask_rows"]
    assert M.sum() == g["mask_count"]
    p = canonical_plan(g["L"], g["window"], g["global_idx"], np.asarray(g["extra_idx"]).reshape(-1, 2), g["block"])
    assert p.bsr_row_ptr.tolist() == g["bsr_row_ptr"]
    assert p.bsr_col.tolist() == g["bsr_col"]
    assert p.tile_masks.reshape(p.n_tiles, -1).tolist() == g["tile_mask_words"]
    assert int(p.tile_popcount().sum()) == g["tile_popcount"]
    assert p.csr_row_ptr.tolist() == g["csr_row_ptr"]
    assert p.csr_col.tolist() == g["csr_col"]
    assert p.global_rows.tolist() == g["global_rows"]


# ---------------------------------------------------------------- brute force
def brute_force_plan(L, window, G, E, b):
    """Element-by-element statement of O-2/O-3 with plain Python loops (tiny L only)."""
    w1 = window // 2
    Gs = set(int(x) for x in np.asarray(G).reshape(-1))
    Es = set((int(r), int(c)) for r, c in np.asarray(E).reshape(-1, 2))

    def M(r, c):
        return abs(r - c) <= w1 or r in Gs or c in Gs or (r, c) in Es

    nb = -(-L // b)
    T = set()
    for r in range(L):
        if r in Gs:
            continue
        for c in range(L):
            if abs(r - c) <= w1:
                T.add((r // b, c // b))
    row_ptr, cols, words = [0], [], []
    wpr = -(-b // 64)
    for I in range(nb):
        for J in range(nb):
            if (I, J) not in T:
                continue
            cols.append(J)
            tw = []
            for a in range(b):
                ws = [0] * wpr
                for beta in range(b):
                    r, c = I * b + a, J * b + beta
                    if r < L and c < L and r not in Gs and M(r, c):
                        ws[beta // 64] |= 1 << (beta % 64)
                tw.extend(ws)
            words.append(tw)
        row_ptr.append(len(cols))
    csr_ptr, csr = [0], []
    for r in range(L):
        if r not in Gs:
            for c in range(L):
                if M(r, c) and (r // b, c // b) not in T:
                    csr.append(c)
        csr_ptr.append(len(csr))
    return row_ptr, cols, words, csr_ptr, csr, sorted(Gs)


@pytest.mark.parametrize("seed", range(40))
def test_plan_brute_force_tiny(seed):
    rng = np.random.default_rng(1000 + seed)
    L, window, G, E = random_small_config(rng, 40)
    b = int(rng.choice([1, 2, 3, 4, 8]))
    p = canonical_plan(L, window, G, E, b)
    row_ptr, cols, words, csr_ptr, csr, gl = brute_force_plan(L, window, G, E, b)
    assert p.bsr_row_ptr.tolist() == row_ptr
    assert p.bsr_col.tolist() == cols
    assert p.tile_masks.reshape(p.n_tiles, -1).tolist() == words
    assert p.csr_row_ptr.tolist() == csr_ptr
    assert p.csr_col.tolist() == csr
    assert p.global_rows.tolist() == gl


def test_plan_brute_force_b64_ragged():
    rng = np.random.default_rng(7)
    L, window = 150, 40
    G = np.array([3, 77, 149])
    E = rng.integers(0, L, size=(200, 2))
    p = canonical_plan(L, window, G, E, 64)
    row_ptr, cols, words, csr_ptr, csr, gl = brute_force_plan(L, window, G, E, 64)
    assert p.bsr_row_ptr.tolist() == row_ptr and p.bsr_col.tolist() == cols
    assert p.tile_masks.reshape(p.n_tiles, -1).astype(np.uint64).tolist() == words
    assert p.csr_row_ptr.tolist() == csr_ptr and p.csr_col.tolist() == csr


# ---------------------------------------------------------------- invariants
def check_invariants(L, window, G, E, b):
    M = union_mask_dense(L, window, G, E)
    p = canonical_plan(L, window, G, E, b)
    cover = np.zeros((L, L), dtype=np.int32)
    for I in range(p.nb):
        for t in range(p.bsr_row_ptr[I], p.bsr_row_ptr[I + 1]):
            J = p.bsr_col[t]
            bits = p.tile_bits(t)
            r1, c1 = min(L, I * b + b) - I * b, min(L, J * b + b) - J * b
            assert not bits[r1:].any() and not bits[:, c1:].any()      # nothing outside [0, L)
            cover[I * b:I * b + r1, J * b:J * b + c1] += bits[:r1, :c1]
    for r in range(L):
        for c in p.csr_col[p.csr_row_ptr[r]:p.csr_row_ptr[r + 1]]:
            cover[r, c] += 1
    cover[p.global_rows, :] += 1
    assert cover.max() <= 1                                # pairwise disjoint
    assert np.array_equal(cover.astype(bool), M)           # exactly the union
    assert p.tile_popcount().sum() + p.csr_col.size + len(p.global_rows) * L == M.sum()


@pytest.mark.parametrize("seed", range(20))
def test_plan_invariants_random(seed):
    rng = np.random.default_rng(seed)
    L, window, G, E = random_small_config(rng, 64)
    check_invariants(L, window, G, E, int(rng.choice([2, 4, 8, 16])))


def test_plan_invariants_c1_both_blocks():
    c = get_config("C1")
    for b in (64, 128):
        check_invariants(c.L, c.window, c.global_idx, c.extra_idx, b)


def test_set_semantics_and_permutation():
    rng = np.random.default_rng(3)
    L, window = 200, 20
    G = np.array([5, 150, 5, 9])
    E = rng.integers(0, L, size=(300, 2))
    p1 = canonical_plan(L, window, G, E, 64)
    E2 = np.concatenate([E[rng.permutation(len(E))], E[:50]])
    p2 = canonical_plan(L, window, np.array([9, 150, 5]), E2, 64)
    for f in ("bsr_row_ptr", "bsr_col", "tile_masks", "csr_row_ptr", "csr_col", "global_rows"):
        assert np.array_equal(getattr(p1, f), getattr(p2, f)), f


def test_global_rows_cleared_and_csr_outside_tiles():
    c = get_config("C3")
    p = canonical_plan(c.L, c.window, c.global_idx, c.extra_idx, 128)
    b = p.block
    g = set(p.global_rows.tolist())
    for I in range(p.nb):
        Js = set(p.bsr_col[p.bsr_row_ptr[I]:p.bsr_row_ptr[I + 1]].tolist())
        for t in range(p.bsr_row_ptr[I], p.bsr_row_ptr[I + 1]):
            bits = p.tile_bits(t)
            for a in range(b):
                if I * b + a in g:
                    assert not bits[a].any()
        for r in range(I * b, min(c.L, I * b + b)):
            for col in p.csr_col[p.csr_row_ptr[r]:p.csr_row_ptr[r + 1]]:
                assert col // b not in Js
    # Appendix A of SURVEY.md: C3 at b=128 -> 46 tiles, fine 105,206, dense-row 131,072
    assert p.n_tiles == 46 and p.csr_col.size == 105_206 and len(g) * c.L == 131_072


@pytest.mark.slow
def test_c4_counts():
    c = get_config("C4")
    assert len(c.extra_idx) == 164 * c.L
    p = canonical_plan(c.L, c.window, c.global_idx, c.extra_idx, 128)
    # exact for any seed: band + 164 per row (the residual is drawn outside the band)
    assert p.tile_popcount().sum() + p.csr_col.size == band_nnz(c.L, 256) + 164 * c.L == 11_026_176
    assert p.n_tiles == 634 and p.n_full_tiles() == 382


# ---------------------------------------------------------------- density threshold tau (f-2)
def _tau_brute(L, window, G, E, b, tau):
    """Independent tile classification by density, straight from the union mask."""
    M = union_mask_dense(L, window, G, E)
    g = np.zeros(L, bool)
    g[np.asarray(G, dtype=np.int64)] = True
    Mc = M & ~g[:, None]
    nb = -(-L // b)
    T = set()
    for I in range(nb):
        for J in range(nb):
            if Mc[I * b:(I + 1) * b, J * b:(J + 1) * b].sum() >= tau * b * b:
                T.add((I, J))
    return Mc, T


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("tau", [0.05, 0.3, 0.75, 1.0])
def test_tau_plan_brute_force(seed, tau):
    rng = np.random.default_rng(100 + seed)
    L, window, G, E = random_small_config(rng, 64)
    b = int(rng.choice([2, 4, 8]))
    p = canonical_plan(L, window, G, E, b, tau=tau)
    Mc, T = _tau_brute(L, window, G, E, b, tau)
    got_T = {(I, int(J)) for I in range(p.nb) for J in p.bsr_col[p.bsr_row_ptr[I]:p.bsr_row_ptr[I + 1]]}
    assert got_T == T
    # every union element of a non-global row is in exactly one part
    rebuilt = np.zeros_like(Mc)
    for t in range(p.n_tiles):
        I = int(np.searchsorted(p.bsr_row_ptr, t, side="right") - 1)
        J = int(p.bsr_col[t])
        bits = p.tile_bits(t)
        r1, c1 = min(b, L - I * b), min(b, L - J * b)
        assert not (rebuilt[I * b:I * b + r1, J * b:J * b + c1] & bits[:r1, :c1]).any()
        rebuilt[I * b:I * b + r1, J * b:J * b + c1] |= bits[:r1, :c1]
        assert not bits[r1:].any() and not bits[:, c1:].any()
    for r in range(L):
        cols = p.csr_col[p.csr_row_ptr[r]:p.csr_row_ptr[r + 1]]
        assert not rebuilt[r, cols].any()
        rebuilt[r, cols] = True
    assert np.array_equal(rebuilt, Mc)


def test_tau_one_keeps_only_full_tiles_and_band_rule_differs():
    c = get_config("C1")
    p1 = canonical_plan(c.L, c.window, c.global_idx, c.extra_idx, 64, tau=1.0)
    assert p1.n_tiles == p1.n_full_tiles()
    p0 = canonical_plan(c.L, c.window, c.global_idx, c.extra_idx, 64)
    # C1 at b=64 has no full tile: tau = 1 leaves everything to the CSR
    assert p0.n_full_tiles() == 0 and p1.n_tiles == 0
    assert p1.csr_col.size == p0.tile_popcount().sum() + p0.csr_col.size
