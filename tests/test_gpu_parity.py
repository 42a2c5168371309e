"""GPU parity: the CUDA path (through the C ABI) vs the fp64 oracle on the same seeded inputs.

Bar (BASELINE.json north_star): outputs in bf16/fp16 with fp32 accumulation within max-abs 2e-2
and mean-abs 2e-3 of the fp64 oracle. Element-by-element at sizes the oracle finishes in seconds
(several 128-row tiles and ragged tails); sampled rows at the BASELINE full sizes in the same
launch configuration bench.py times.
"""
import numpy as np
import pytest
import torch

import paper_conf_iiswc_lica22_b200 as mg
from oracle import (ExtraIndex, attention_rows, dense_masked_attention, global_flags, head_inputs_f64)
from workloads import bits_to_f64, get_config, make_qkv, random_residual
from gpu_util import TOL_MAX, TOL_MEAN, err_stats, from_device, to_device

pytestmark = pytest.mark.gpu


def run_gpu(plan, q, k, v, dtype="bf16", layout="bhld"):
    Q, K, V = (to_device(x, dtype) for x in (q, k, v))
    if layout == "blhd":
        # physical [B, L, H, d], passed as a [B, H, L, d] strided view (L x D_m hidden states)
        Q, K, V = (x.transpose(1, 2).contiguous().transpose(1, 2) for x in (Q, K, V))
        O = torch.empty_like(Q.transpose(1, 2)).transpose(1, 2)
    else:
        O = torch.empty_like(Q)
    out = mg.sparse_attention_fwd(plan, Q, K, V, O)
    torch.cuda.synchronize()
    return from_device(out)


def oracle_full(q, k, v, window, G, E, dtype="bf16"):
    B, H, L, d = q.shape
    ref = np.zeros((B, H, L, d))
    for b in range(B):
        for h in range(H):
            Q, K, V = head_inputs_f64(q, k, v, b, h, dtype)
            ref[b, h] = dense_masked_attention(Q, K, V, window, G, E)
    return ref


def check(got, ref, tol_max=TOL_MAX, tol_mean=TOL_MEAN):
    mx, mean = err_stats(got, ref)
    assert np.isfinite(got).all()
    assert mx <= tol_max and mean <= tol_mean, (mx, mean)
    return mx, mean


@pytest.mark.parametrize("dist", ["normal", "peaky", "adversarial"])
def test_c1_full(dist):
    c = get_config("C1")
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=c.seed, dist=dist, global_idx=c.global_idx)
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
    got = run_gpu(plan, q, k, v)
    ref = oracle_full(q, k, v, c.window, c.global_idx, c.extra_idx)
    if dist == "peaky":
        check(got, ref, tol_max=2e-2 * max(1.0, np.abs(ref).max() / 4))
    else:
        check(got, ref)


MIXED = dict(B=2, H=3, L=1024, window=128, G=np.array([0, 1, 2, 130, 777], np.int32))


def mixed_extra(L, seed=3, per_row=6):
    return random_residual(L, 128, per_row, seed=seed)


@pytest.mark.parametrize("fine_kernel,concurrency", [(0, 1), (0, 2), (0, 3), (1, 1)])
@pytest.mark.parametrize("strip", [0, -1])
@pytest.mark.parametrize("all_fine", [False, True])
def test_mixed_pattern_all_parts(strip, all_fine, fine_kernel, concurrency):
    """Band tiles + strip tiles or CSR rows (tensor-core or CUDA-core fine kernel) + dense global
    rows, several heads."""
    m = MIXED
    E = mixed_extra(m["L"])
    q, k, v = make_qkv(m["B"], m["H"], m["L"], 64, seed=5, dist="adversarial", global_idx=m["G"])
    plan = mg.Plan(m["L"], m["H"], 64, m["window"], m["G"], E, strip_max_cols=strip, force_all_fine=all_fine,
                   fine_kernel=fine_kernel, concurrency=concurrency)
    inf = plan.info()
    if all_fine:
        assert inf["n_tiles"] == 0 and inf["nnz_fine_cuda"] == inf["nnz_fine"]
    got = run_gpu(plan, q, k, v)
    ref = oracle_full(q, k, v, m["window"], m["G"], E)
    check(got, ref)


@pytest.mark.parametrize("fine_kernel,concurrency", [(0, 1), (0, 2), (0, 3), (1, 1)])
@pytest.mark.parametrize("dtype", ["bf16", "fp16"])
@pytest.mark.parametrize("dist", ["normal", "peaky", "adversarial"])
def test_fine_rows_all_lengths(fine_kernel, concurrency, dtype, dist):
    """CSR-only rows of every length 1..70 (ragged 16-nnz steps of the tensor-core fine kernel,
    32-index windows, final rows written directly) plus rows with a coarse part (fp32 partials)."""
    L, G = 768, np.array([700], np.int32)
    rng = np.random.default_rng(11)
    pairs = []
    for r in range(L):
        n = 1 + r % 70
        pairs += [(r, c) for c in rng.choice(L, n, replace=False)]
    E = np.array(pairs, np.int32)
    q, k, v = make_qkv(1, 2, L, 64, seed=12, dist=dist, global_idx=G, dtype=dtype)
    for all_fine in (True, False):
        plan = mg.Plan(L, 2, 64, 32, G, E, strip_max_cols=-1, force_all_fine=all_fine, fine_kernel=fine_kernel,
                       concurrency=concurrency)
        assert plan.info()["nnz_fine_cuda"] > 0
        got = run_gpu(plan, q, k, v, dtype=dtype)
        ref = oracle_full(q, k, v, 32, G, E, dtype=dtype)
        check(got, ref, tol_max=2e-2 * max(1.0, np.abs(ref).max() / 4))


@pytest.mark.parametrize("tau", [0.1, 0.5, 1.0])
def test_density_threshold_plans(tau):
    """tau > 0 tile rule (A17): band-edge tiles below the threshold move to the CSR part, dense
    random blocks become coarse; every part still runs and merges correctly."""
    L, G = 1024, np.array([3, 600], np.int32)
    rng = np.random.default_rng(4)
    blocks = [(int(rng.integers(0, 16)), int(rng.integers(0, 16))) for _ in range(10)]
    E = np.array([(I * 64 + a, J * 64 + c) for I, J in blocks for a in range(64) for c in range(64)], np.int32)
    E = np.concatenate([E, random_residual(L, 96, 5, seed=6)])
    q, k, v = make_qkv(2, 2, L, 64, seed=13, dist="adversarial", global_idx=G)
    plan = mg.Plan(L, 2, 64, 96, G, E, tau=tau)
    check(run_gpu(plan, q, k, v), oracle_full(q, k, v, 96, G, E))


@pytest.mark.parametrize("dense_chunk", [-1, 1, 3, 8])
@pytest.mark.parametrize("L,G", [(1024, list(range(40))), (1000, [0, 5, 999]), (640, list(range(0, 640, 4)))])
def test_dense_row_split_chunks(dense_chunk, L, G):
    """Global rows split over column-tile chunks (a-4) merged by the last chunk; repeated calls keep
    the per-group counters consistent; >128 global rows give several row groups."""
    G = np.array(G, np.int32)
    q, k, v = make_qkv(2, 3, L, 64, seed=31, dist="adversarial", global_idx=G)
    plan = mg.Plan(L, 3, 64, 64, G, None, dense_chunk=dense_chunk)
    ref = oracle_full(q, k, v, 64, G, np.zeros((0, 2), np.int32))
    for _ in range(3):
        check(run_gpu(plan, q, k, v), ref)


def test_strip_path_c2_pattern_small():
    """C2-like globals [0, 32) with fewer blocks: the CSR residual runs as tensor-core strips."""
    L, G = 1024, np.arange(32, dtype=np.int32)
    plan = mg.Plan(L, 2, 64, 256, G, None)
    inf = plan.info()
    assert inf["nnz_fine_strip"] == inf["nnz_fine"] > 0 and inf["n_strip_tiles"] > 0
    q, k, v = make_qkv(1, 2, L, 64, seed=9, dist="adversarial", global_idx=G)
    check(run_gpu(plan, q, k, v), oracle_full(q, k, v, 256, G, np.zeros((0, 2))))


@pytest.mark.parametrize("L,window,G", [(1000, 64, [0, 999]), (300, 40, [5]), (129, 0, []), (64, 16, [3]),
                                        (200, 512, [])])
def test_ragged_lengths(L, window, G):
    E = np.random.default_rng(L).integers(0, L, size=(3 * L, 2)).astype(np.int32)
    q, k, v = make_qkv(2, 2, L, 64, seed=L)
    plan = mg.Plan(L, 2, 64, window, G, E)
    check(run_gpu(plan, q, k, v), oracle_full(q, k, v, window, G, E))


def test_blhd_layout():
    m = MIXED
    E = mixed_extra(m["L"], seed=8)
    q, k, v = make_qkv(m["B"], m["H"], m["L"], 64, seed=2)
    plan = mg.Plan(m["L"], m["H"], 64, m["window"], m["G"], E)
    check(run_gpu(plan, q, k, v, layout="blhd"), oracle_full(q, k, v, m["window"], m["G"], E))


def test_fp16():
    c = get_config("C1")
    q, k, v = make_qkv(1, 2, c.L, 64, seed=4, dtype="fp16")
    plan = mg.Plan(c.L, 2, 64, c.window, c.global_idx, c.extra_idx)
    got = run_gpu(plan, q, k, v, dtype="fp16")
    check(got, oracle_full(q, k, v, c.window, c.global_idx, c.extra_idx, dtype="fp16"))


def test_diagonal_only_is_identity():
    L = 512
    q, k, v = make_qkv(1, 2, L, 64, seed=1)
    plan = mg.Plan(L, 2, 64, 0, [], None)
    got = run_gpu(plan, q, k, v)
    assert np.array_equal(got, bits_to_f64(v))          # P = 1 on the diagonal: exact


def test_ones_v_and_zero_q():
    c = get_config("C1")
    q, k, v = make_qkv(1, 1, c.L, 64, seed=1, dist="ones_v")
    plan = mg.Plan(c.L, 1, 64, c.window, c.global_idx, c.extra_idx)
    got = run_gpu(plan, q, k, v)
    assert np.abs(got - 1.0).max() <= 2 ** -7
    q, k, v = make_qkv(1, 1, c.L, 64, seed=1, dist="zeros_q")
    check(run_gpu(plan, q, k, v), oracle_full(q, k, v, c.window, c.global_idx, c.extra_idx))


def test_concurrent_repeat_calls_and_batch_change():
    """Concurrent mode: per-row counters stay consistent over repeated calls and batch changes."""
    m = MIXED
    E = mixed_extra(m["L"], seed=9)
    plan = mg.Plan(m["L"], m["H"], 64, m["window"], m["G"], E, strip_max_cols=-1, concurrency=2)
    for B in (2, 3, 1, 3):
        q, k, v = make_qkv(B, m["H"], m["L"], 64, seed=B)
        ref = oracle_full(q, k, v, m["window"], m["G"], E)
        for _ in range(2):
            check(run_gpu(plan, q, k, v), ref)


def test_repeat_calls_deterministic_and_batch_growth():
    c = get_config("C1")
    plan = mg.Plan(c.L, 1, 64, c.window, c.global_idx, c.extra_idx)
    q, k, v = make_qkv(1, 1, c.L, 64, seed=3)
    a = run_gpu(plan, q, k, v)
    b = run_gpu(plan, q, k, v)
    assert np.array_equal(a, b)
    q4, k4, v4 = make_qkv(4, 1, c.L, 64, seed=3)     # workspace grows with the batch
    check(run_gpu(plan, q4, k4, v4), oracle_full(q4, k4, v4, c.window, c.global_idx, c.extra_idx))


def test_invalid_tensor_args():
    c = get_config("C1")
    plan = mg.Plan(c.L, 1, 64, c.window, c.global_idx, c.extra_idx)
    Q = torch.zeros(1, 1, c.L, 64, dtype=torch.bfloat16, device="cuda")
    with pytest.raises(mg.MGError):                     # heads mismatch
        mg.sparse_attention_fwd(plan, Q.expand(1, 2, c.L, 64), Q, Q)
    with pytest.raises(mg.MGError):                     # dtype mismatch
        mg.sparse_attention_fwd(plan, Q, Q.half(), Q)
    with pytest.raises(mg.MGError):                     # seq_len mismatch
        Z = torch.zeros(1, 1, c.L - 8, 64, dtype=torch.bfloat16, device="cuda")
        mg.sparse_attention_fwd(plan, Z, Z, Z)


def test_host_entry_point_matches_device():
    m = MIXED
    E = mixed_extra(m["L"], seed=4)
    q, k, v = make_qkv(m["B"], m["H"], m["L"], 64, seed=6)
    plan = mg.Plan(m["L"], m["H"], 64, m["window"], m["G"], E)
    dev = run_gpu(plan, q, k, v)
    h = [torch.from_numpy(x.view(np.int16)).view(torch.bfloat16).pin_memory() for x in (q, k, v)]
    O = torch.empty_like(h[0]).pin_memory()
    mg.sparse_attention_fwd_host(plan, h[0], h[1], h[2], O)
    torch.cuda.synchronize()
    assert np.array_equal(from_device(O), dev)


# ------------------------------------------------------------------ full BASELINE sizes (sampled)
def sample_rows(L, G, rng, n=48):
    rows = set(rng.choice(L, n, replace=False).tolist())
    rows |= {0, 1, 127, 128, L - 1, L - 128}
    rows |= set(np.asarray(G)[:4].tolist())
    return sorted(r for r in rows if 0 <= r < L)


@pytest.mark.parametrize("cfg,fine_kernel,concurrency", [("C2", 0, 0), ("C3", 0, 0), ("C4", 0, 1), ("C4", 0, 2), ("C4", 0, 3),
                                                          ("C4", 1, 1), ("QDS-LS", 0, 0), ("F9-LS", 0, 0),
                                                          ("F9-LSG", 0, 0), ("F9-LBR", 0, 0), ("F9-RBR", 0, 0),
                                                          ("F9-RBR", 0, 0.2)])
def test_full_size_sampled(cfg, fine_kernel, concurrency):
    c = get_config(cfg)
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=c.seed)
    # (a float in the concurrency column is a tau for the density tile rule, with the default mode)
    tau = concurrency if isinstance(concurrency, float) else 0.0
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx, fine_kernel=fine_kernel,
                   concurrency=0 if tau else concurrency, tau=tau)
    got = run_gpu(plan, q, k, v)
    assert np.isfinite(got).all()
    rng = np.random.default_rng(17)
    g = global_flags(c.L, c.global_idx)
    ex = ExtraIndex(c.L, c.extra_idx)
    errs = []
    for (b, h) in [(0, 0), (c.B - 1, c.H - 1), (c.B // 2, 1)]:
        rows = sample_rows(c.L, c.global_idx, rng)
        Q, K, V = head_inputs_f64(q, k, v, b, h)
        ref = attention_rows(Q, K, V, rows, c.window, g, ex)
        errs.append(np.abs(got[b, h, rows] - ref))
    e = np.concatenate(errs)
    assert e.max() <= TOL_MAX and e.mean() <= TOL_MEAN, (e.max(), e.mean())


# ------------------------------------------------------------------ padding (valid length, A18)
@pytest.mark.parametrize("case", ["mixed", "c1", "fine_only", "dense_split", "concurrent", "sm_split"])
def test_padded_batch(case):
    """mg_sparse_attention_fwd_padded: per-sample valid lengths (including 0, full, and cuts inside
    row blocks and strips); every part (tiles, strips, CSR rows, dense rows, split dense chunks,
    concurrent merge) masks the padded columns and zeroes the padded rows."""
    if case == "c1":
        c = get_config("C1")
        B, H, L, window, G, E = 4, 1, c.L, c.window, c.global_idx, c.extra_idx
        kw = {}
    else:
        m = MIXED
        B, H, L, window, G = 4, m["H"], m["L"], m["window"], m["G"]
        E = mixed_extra(L, seed=12)
        kw = {"fine_only": dict(strip_max_cols=-1), "dense_split": dict(dense_chunk=2),
              "concurrent": dict(strip_max_cols=-1, concurrency=2),
              "sm_split": dict(strip_max_cols=-1, concurrency=3), "mixed": {}}[case]
    q, k, v = make_qkv(B, H, L, 64, seed=41, dist="adversarial", global_idx=G)
    plan = mg.Plan(L, H, 64, window, G, E, **kw)
    lens = np.array([L, 0, L // 2 + 37, 129][:B], np.int32)
    Q, K, V = (to_device(x) for x in (q, k, v))
    vl = torch.from_numpy(lens).cuda()
    got = from_device(mg.sparse_attention_fwd_padded(plan, Q, K, V, vl))
    for b in range(B):
        for h in range(H):
            Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
            ref = dense_masked_attention(Qh, Kh, Vh, window, G, E, valid_len=int(lens[b]))
            mx, mean = err_stats(got[b, h], ref)
            # adversarial inputs: bf16 output rounding grows with |O| (as for the peaky case)
            assert mx <= TOL_MAX * max(1.0, np.abs(ref).max() / 4) and mean <= TOL_MEAN, (case, b, h, mx, mean)
            assert (got[b, h, lens[b]:] == 0).all()


# ------------------------------------------------------------------ batched plans (per-sample positions)
@pytest.mark.parametrize("kw", [{}, dict(strip_max_cols=-1), dict(strip_max_cols=-1, concurrency=2),
                                dict(strip_max_cols=-1, concurrency=3), dict(fine_kernel=1, strip_max_cols=-1)])
def test_batched_plan_per_sample_positions(kw):
    """One launch over a batch whose samples have different global tokens and residuals (P:66,
    P:94), against the oracle per sample; padded too."""
    L, H, w = 1024, 2, 128
    rng = np.random.default_rng(51)
    Gs = [np.array([0, 5, 700], np.int32), np.array([300], np.int32), np.zeros(0, np.int32),
          np.arange(0, 40, dtype=np.int32)]
    Es = [random_residual(L, w, int(rng.integers(0, 6)), seed=60 + b) for b in range(4)]
    plan = mg.BatchedPlan(L, H, 64, w, Gs, Es, **kw)
    q, k, v = make_qkv(4, H, L, 64, seed=52)
    got = run_gpu(plan, q, k, v)
    lens = np.array([L, 333, 1000, 129], np.int32)
    Q, K, V = (to_device(x) for x in (q, k, v))
    gotp = from_device(mg.sparse_attention_fwd_padded(plan, Q, K, V, torch.from_numpy(lens).cuda()))
    for b in range(4):
        for h in range(H):
            Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
            check(got[b, h], dense_masked_attention(Qh, Kh, Vh, w, Gs[b], Es[b]))
            check(gotp[b, h], dense_masked_attention(Qh, Kh, Vh, w, Gs[b], Es[b], valid_len=int(lens[b])))
    with pytest.raises(mg.MGError):                 # batch must match the plan's samples
        run_gpu(plan, q[:2], k[:2], v[:2])


def test_fine_tma_gather_variant_subprocess():
    """The TMA tile::gather4 variant of the two-head fine kernel (off by default, MG_FINE_TMA=1)
    against the oracle, in a subprocess (the switch is read once per process)."""
    import os
    import subprocess
    import sys
    code = (
        "import numpy as np, sys; sys.path.insert(0, 'tests');"
        "import paper_conf_iiswc_lica22_b200 as mg;"
        "from gpu_util import from_device, to_device, err_stats;"
        "from oracle import dense_masked_attention, head_inputs_f64;"
        "from workloads import make_qkv, random_residual;"
        "L, H, W = 1024, 4, 128; G = np.array([0, 300], np.int32); E = random_residual(L, W, 9, seed=3);"
        "q, k, v = make_qkv(2, H, L, 64, seed=5);"
        "plan = mg.Plan(L, H, 64, W, G, E, strip_max_cols=-1);"
        "got = from_device(mg.sparse_attention_fwd(plan, *(to_device(x) for x in (q, k, v))));"
        "w = max(err_stats(got[b, h], dense_masked_attention(*head_inputs_f64(q, k, v, b, h), W, G, E))[0]"
        "        for b in range(2) for h in range(H));"
        "assert w <= 2e-2, w; print('ok', w)")
    env = dict(os.environ, MG_FINE_TMA="1")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env, cwd=root, timeout=300)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-2000:]
