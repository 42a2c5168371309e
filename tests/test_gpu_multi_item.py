"""GPU parity of the persistent multi-item regime.

The coarse kernel is persistent: each CTA claims work items from an atomic counter into a 4-deep
ring, double-buffers the items' Q tiles, carries the MMA issuer's pending P.V across item
boundaries and stages O tiles in the Q buffer for TMA stores; the fine kernel's warps walk a
grid-stride row sequence with the gather pointer running ahead across rows. At the small test
sizes a CTA (or a warp) normally sees only one or two items (rows), so these tests shrink the grid
with the plan option num_sms (grid = 2 x num_sms coarse CTAs, resident-blocks x num_sms fine
blocks): every CTA then runs dozens of items and every fine warp dozens of rows. All elements are
compared with the fp64 oracle (O-4) at the north_star bar.
"""
import numpy as np
import pytest
import torch

import paper_conf_iiswc_lica22_b200 as mg
from oracle import dense_masked_attention, head_inputs_f64
from workloads import get_config, make_qkv, random_residual
from gpu_util import TOL_MAX, TOL_MEAN, err_stats, from_device, to_device

pytestmark = pytest.mark.gpu

L, H, B, W = 1024, 3, 2, 128
G = np.array([0, 1, 2, 130, 777], np.int32)


def oracle_all(q, k, v, window, Gs, Es, lens=None):
    Bq, Hq = q.shape[:2]
    out = np.zeros(q.shape, np.float64)
    for b in range(Bq):
        for h in range(Hq):
            Q, K, V = head_inputs_f64(q, k, v, b, h)
            g = Gs[b] if isinstance(Gs, list) else Gs
            e = Es[b] if isinstance(Es, list) else Es
            out[b, h] = dense_masked_attention(Q, K, V, window, g, e,
                                               valid_len=None if lens is None else int(lens[b]))
    return out


def check(got, ref):
    mx, mean = err_stats(got, ref)
    assert np.isfinite(got).all()
    # adversarial inputs: bf16 output rounding grows with |O| (tolerance scale as in test_gpu_parity)
    assert mx <= TOL_MAX * max(1.0, np.abs(ref).max() / 4) and mean <= TOL_MEAN, (mx, mean)


@pytest.mark.parametrize("num_sms", [1, 2, 3])
@pytest.mark.parametrize("kw", [{}, dict(strip_max_cols=-1), dict(strip_max_cols=-1, concurrency=2),
                                dict(strip_max_cols=-1, concurrency=3), dict(dense_chunk=2), dict(force_all_fine=True)],
                         ids=["strips", "csr_rows", "concurrent", "sm_split", "dense_split", "all_fine"])
def test_few_ctas_many_items(num_sms, kw):
    E = random_residual(L, W, 6, seed=3)
    q, k, v = make_qkv(B, H, L, 64, seed=5, dist="adversarial", global_idx=G)
    plan = mg.Plan(L, H, 64, W, G, E, num_sms=num_sms, **kw)
    ref = oracle_all(q, k, v, W, G, E)
    Q, K, V = (to_device(x) for x in (q, k, v))
    for _ in range(2):   # the self-resetting work counter and split-dense counters across calls
        check(from_device(mg.sparse_attention_fwd(plan, Q, K, V)), ref)


@pytest.mark.parametrize("num_sms", [1, 3])
def test_few_ctas_padded_and_batched(num_sms):
    Gs = [np.array([0, 5, 700], np.int32), np.array([300], np.int32), np.zeros(0, np.int32),
          np.arange(0, 40, dtype=np.int32)]
    Es = [random_residual(L, W, b + 1, seed=60 + b) for b in range(4)]
    plan = mg.BatchedPlan(L, 2, 64, W, Gs, Es, num_sms=num_sms)
    q, k, v = make_qkv(4, 2, L, 64, seed=52)
    Q, K, V = (to_device(x) for x in (q, k, v))
    check(from_device(mg.sparse_attention_fwd(plan, Q, K, V)), oracle_all(q, k, v, W, Gs, Es))
    lens = np.array([L, 333, 1000, 129], np.int32)
    got = from_device(mg.sparse_attention_fwd_padded(plan, Q, K, V, torch.from_numpy(lens).cuda()))
    check(got, oracle_all(q, k, v, W, Gs, Es, lens))
    # single-sample plan, padded, with split dense chunks and CSR rows
    E = random_residual(L, W, 4, seed=9)
    plan = mg.Plan(L, 2, 64, W, G, E, num_sms=num_sms, strip_max_cols=-1, dense_chunk=3)
    got = from_device(mg.sparse_attention_fwd_padded(plan, Q, K, V, torch.from_numpy(lens).cuda()))
    check(got, oracle_all(q, k, v, W, G, E, lens))


def test_fine_warps_walk_many_rows():
    """C4-like random residual with one SM's worth of fine warps: every warp walks ~100 rows of
    different lengths, so the gather pointer's cross-row run-ahead is exercised on every row."""
    Lr = 2048
    rng = np.random.default_rng(21)
    pairs = []
    for r in range(Lr):
        n = int(rng.integers(1, 60))
        cand = np.array([c for c in range(Lr) if abs(c - r) > 64])
        pairs += [(r, int(c)) for c in rng.choice(cand, n, replace=False)]
    E = np.array(pairs, np.int32)
    q, k, v = make_qkv(1, 2, Lr, 64, seed=22)
    Q, K, V = (to_device(x) for x in (q, k, v))
    ref = oracle_all(q, k, v, 128, np.zeros(0, np.int32), E)
    for kw in (dict(), dict(force_all_fine=True)):
        plan = mg.Plan(Lr, 2, 64, 128, [], E, num_sms=1, **kw)
        assert plan.info()["nnz_fine_cuda"] > 0
        check(from_device(mg.sparse_attention_fwd(plan, Q, K, V)), ref)


def test_c2_full_batch_element_all_heads():
    """Full-size C2 (the bench workload, default launch configuration): every element of all 12
    heads of one batch element against the fp64 oracle (the other 7 elements run in the same
    launch; their first and last heads are checked too)."""
    c = get_config("C2")
    q, k, v = make_qkv(c.B, c.H, c.L, c.d, seed=c.seed)
    plan = mg.Plan(c.L, c.H, c.d, c.window, c.global_idx, c.extra_idx)
    Q, K, V = (to_device(x) for x in (q, k, v))
    got = from_device(mg.sparse_attention_fwd(plan, Q, K, V))
    assert np.isfinite(got).all()
    heads = [(c.B // 2, h) for h in range(c.H)] + [(c.B - 1, 0), (c.B - 1, c.H - 1), (0, 0)]
    errs = []
    for b, h in heads:
        Qh, Kh, Vh = head_inputs_f64(q, k, v, b, h)
        ref = dense_masked_attention(Qh, Kh, Vh, c.window, c.global_idx, c.extra_idx)
        errs.append(np.abs(got[b, h] - ref))
    e = np.stack(errs)
    assert e.max() <= TOL_MAX and e.mean() <= TOL_MEAN, (e.max(), e.mean())


def test_host_entry_point_seq_first_layout():
    """mg_sparse_attention_fwd_host with physical [L, B, H, d] host tensors (batch not outermost):
    the batch-chunked copy pipeline must fall back to one span."""
    E = random_residual(L, W, 4, seed=4)
    q, k, v = make_qkv(B, H, L, 64, seed=6)
    plan = mg.Plan(L, H, 64, W, G, E)
    host = [torch.from_numpy(np.ascontiguousarray(x.transpose(2, 0, 1, 3)).view(np.int16)).view(torch.bfloat16)
            for x in (q, k, v)]                                  # [L, B, H, d] physical
    host = [h.pin_memory().permute(1, 2, 0, 3) for h in host]    # [B, H, L, d] view, stride_b = H*d
    O = torch.empty(L, B, H, 64, dtype=torch.bfloat16).pin_memory().permute(1, 2, 0, 3)
    mg.sparse_attention_fwd_host(plan, host[0], host[1], host[2], O)
    torch.cuda.synchronize()
    check(from_device(O), oracle_all(q, k, v, W, G, E))
