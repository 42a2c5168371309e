"""Benchmark of the Multigrain compound sparse attention forward on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C2|C5|...] [--impl mine|reference]

One "step" = one mg_sparse_attention_fwd over one batch of the workload (every hot-path step:
plan already built, SDDMM -> merged SpSoftmax -> SpMM over the coarse, fine and dense-row parts).
N=1 default workload: C2 (Longformer-base L=4096, H=12, B=8, w=512, 32 global tokens) —
BASELINE.json configs[1], the config its metric is quoted on. N>1 default (torchrun, one process
per GPU): C5, BASELINE.json configs[4] — the C2 pattern at a global batch of 64 sharded over the
ranks in contiguous batch slices (dist.shard_range, B/n per rank; strong scaling). The (b, h)
units are independent, so there is no data-path collective; an NCCL all_gather of O
(north_star: gather outputs in the scaling bench) is timed separately. `--workload C5 --gpus 1`
gives the single-GPU time T1 of the sweep; efficiency T1 / (n Tn) is left to the driver. Any other
workload at N>1 runs weak (each rank its own seeded batch).

Timing: W untimed warm-up steps; the K timed steps are bracketed by barrier + synchronize; each
step is preceded by a 256 MB L2 flush (outside its CUDA-event pair) and timed by the library's
CUDA events on the launching stream (mg_plan_get_profile_calls: mean, median, min per step);
max over ranks. value = useful TFLOP/s of the whole job, useful flops = 4 * nnz(M) * d * B * H
(SURVEY.md §8(d)).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "sparse-attn fwd ms and useful TFLOP/s per B200 (Longformer L=4096), 1/2/4/8 GPU"
UNIT = "TFLOP/s"
FALLBACK_PEAKS = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}
# L2 -> SM gather ceiling measured on B200 (tools/microbench/gather_bw.cu: 8 lanes per 128-B row,
# 16-B register loads, no arithmetic), the honest roofline of the L2-served fine kernel
L2_GATHER_GBS = 22200.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--workload", default=None,
                    choices=["C1", "C2", "C3", "C4", "C5", "QDS-LS", "F9-LS", "F9-LSG", "F9-LBR", "F9-RBR", "DIL-LD"],
                    help="default: C2 at N=1, C5 (strong scaling, global batch 64) at N>1")
    ap.add_argument("--impl", default="mine", choices=["mine", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=30)
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="CPU oracle sample budget")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--strip-max-cols", type=int, default=0)
    ap.add_argument("--ablation", action="store_true",
                    help="also time the staged paper-dataflow forward (mg_sparse_attention_fwd_staged)")
    ap.add_argument("--concurrency", type=int, default=0, choices=[0, 1, 2, 3],
                    help="coarse vs CSR kernels: 0 = library default, 1 = serial, 2 = concurrent streams, 3 = SM split")
    ap.add_argument("--tau", type=float, default=0.0, help="tile density threshold (0 = band rule)")
    ap.add_argument("--block", type=int, default=0, choices=[0, 64, 128], help="plan block size (0 = 128)")
    ap.add_argument("--head-dim", type=int, default=0, choices=[0, 64, 128],
                    help="head dimension override (0 = the workload's, 64); 128 for the d = 128 line")
    ap.add_argument("--dense-chunk", type=int, default=0, help="column tiles per dense-row item (-1: no split)")
    ap.add_argument("--fine-kernel", type=int, default=0, choices=[0, 1],
                    help="CSR rows: 0 = warp-level tensor-core kernel, 1 = CUDA-core kernel (A/B)")
    return ap.parse_args()


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured (MEASURED_PEAKS.json)"
    return dict(FALLBACK_PEAKS), "fallback (B200_PROFILING.md)"


def resolve_workload(args, world):
    return args.workload or ("C2" if world == 1 else "C5")


# ------------------------------------------------------------------ sharding (host logic; gloo-tested)
def shard_for_rank(cfg, world: int, rank: int, strong: bool):
    """Batch rows [lo, hi) of the global batch this rank computes. Strong scaling (C5): the global
    batch cfg.B is split into contiguous slices (dist.shard_range: the (b, h) units are
    independent). Weak scaling: every rank computes its own batch of cfg.B."""
    from paper_conf_iiswc_lica22_b200.dist import shard_range
    if strong:
        return shard_range(cfg.B, world, rank)
    return 0, cfg.B


def batch_inputs(cfg, lo: int, hi: int, rank: int, strong: bool):
    """Q, K, V bit patterns [hi - lo, H, L, d] of the rank's slice. Strong scaling draws every batch
    element from its own seed (cfg.seed + 1000 b), so a slice does not depend on the world size and
    the gathered output equals the single-GPU output of the global batch element for element."""
    import numpy as np
    from paper_conf_iiswc_lica22_b200.dist import rank_seed
    from workloads import make_qkv
    if not strong:
        return make_qkv(cfg.B, cfg.H, cfg.L, cfg.d, seed=rank_seed(cfg.seed, rank))
    parts = [make_qkv(1, cfg.H, cfg.L, cfg.d, seed=cfg.seed + 1000 * b) for b in range(lo, hi)]
    if not parts:
        z = np.zeros((0, cfg.H, cfg.L, cfg.d), np.uint16)
        return z, z.copy(), z.copy()
    return tuple(np.concatenate([p[i] for p in parts]) for i in range(3))


def gather_output(O_local, global_batch: int, strong: bool):
    """The scaling bench's only collective: all_gather of O (strong: reassembled [global_batch, ...]
    in batch order; weak: [world, B, ...])."""
    from paper_conf_iiswc_lica22_b200.dist import gather_batches, gather_outputs
    return gather_batches(O_local, global_batch) if strong else gather_outputs(O_local)


def workload_config(cfg, n_gpus, strong, b_local):
    return {
        "workload": f"{cfg.name}: {cfg.note}",
        "B_per_gpu": b_local, "H": cfg.H, "L": cfg.L, "d": cfg.d, "window": cfg.window,
        "n_global": int(len(cfg.global_idx)), "n_extra": int(len(cfg.extra_idx)),
        "global_batch": cfg.B if strong else cfg.B * n_gpus,
        "parallelism": (f"{n_gpus} rank(s), global batch sharded in contiguous slices (strong), no data-path collective"
                        if strong else f"{n_gpus} rank(s), one batch per rank (weak), no data-path collective"),
        "l2": "256 MB L2 flush written before every timed step (outside the event pair)",
        "inputs": ("Q,K,V ~ N(0,1) -> bf16 (workloads.make_qkv, seed 1000*b per batch element)" if strong
                   else "Q,K,V ~ N(0,1) -> bf16 (workloads.make_qkv, seed 0 + 1000*rank)"),
    }


# ------------------------------------------------------------------ clocks (NVML, during the region)
class ClockSampler:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device_index: int, period_s: float = 0.002):
        self.ok = False
        self.samples, self.reasons = [], 0
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # noqa: BLE001
            self.err = str(e)
        self.period = period_s
        self._stop = threading.Event()

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                try:
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                except AttributeError:
                    r = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                self.reasons |= int(r)
            except Exception:  # noqa: BLE001
                pass
            time.sleep(self.period)

    def start(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()

    def stop(self):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "")}
        reasons = [n for bit, n in self.REASONS.items() if self.reasons & bit and bit != 0x1]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": reasons, "samples": len(self.samples)}


def nvml_index(local: int) -> int:
    """NVML (physical) index of the local CUDA device, honouring CUDA_VISIBLE_DEVICES."""
    vis = os.environ.get("CUDA_VISIBLE_DEVICES")
    if vis:
        ids = [x.strip() for x in vis.split(",") if x.strip()]
        if local < len(ids) and ids[local].isdigit():
            return int(ids[local])
    return local


# ------------------------------------------------------------------ CPU oracle baseline
def _oracle_unit(args):
    """One (b, h) unit of the CPU baseline: the oracle's dense masked attention (O-4, fp64)."""
    from threadpoolctl import threadpool_limits
    from oracle import dense_masked_attention
    from workloads import bits_to_f64
    q, k, v, window, g, e = args
    with threadpool_limits(1):   # one core per worker process (the pool provides the parallelism)
        dense_masked_attention(bits_to_f64(q), bits_to_f64(k), bits_to_f64(v), window, g, e)
    return 1


def cpu_oracle_pool(cfg, budget_s: float):
    """The oracle as it stands (never tuned) over the workload's (b, h) units with a process pool of
    os.cpu_count() single-threaded workers, until every unit is done or the budget is spent."""
    import multiprocessing as mp
    from oracle import ExtraIndex, global_flags
    from oracle.mask import mask_row_cols
    from workloads import make_qkv
    g, ex = global_flags(cfg.L, cfg.global_idx), ExtraIndex(cfg.L, cfg.extra_idx)
    nnz = sum(mask_row_cols(r, cfg.L, cfg.window, g, ex).size for r in range(cfg.L))
    q, k, v = make_qkv(cfg.B, cfg.H, cfg.L, cfg.d, seed=cfg.seed)
    units = [(q[b, h], k[b, h], v[b, h], cfg.window, cfg.global_idx, cfg.extra_idx)
             for b in range(cfg.B) for h in range(cfg.H)]
    cores = os.cpu_count() or 1
    ctx = mp.get_context("spawn")
    with ctx.Pool(cores) as pool:
        pool.map(_oracle_unit, units[:cores])          # warm the workers (imports), untimed
        done, t0 = 0, time.perf_counter()
        for _ in pool.imap(_oracle_unit, units, chunksize=1):
            done += 1
            if time.perf_counter() - t0 > budget_s and done % cores == 0:
                break
        dt = time.perf_counter() - t0
        pool.terminate()
    return {"value": 4.0 * nnz * cfg.d * done / dt / 1e12, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"oracle.dense_masked_attention (fp64 numpy) on {done} of {len(units)} (b,h) units of "
                      f"{cfg.name} ({'all' if done == len(units) else 'a bounded sample'}), process pool of "
                      f"{cores} single-threaded workers, {dt:.1f} s wall; useful flops counted as for the GPU"}


_REF = {}


def _ref_init(name, head_dim, seed_heads):
    """Worker initializer of the reference arm: the workload's pattern and a few (b, h) heads of
    seeded inputs, built once per worker process."""
    import dataclasses
    from oracle import ExtraIndex, global_flags, head_inputs_f64
    from workloads import get_config, make_qkv
    from threadpoolctl import threadpool_limits
    threadpool_limits(1)
    cfg = get_config(name)
    if head_dim:
        cfg = dataclasses.replace(cfg, d=head_dim)
    q, k, v = make_qkv(1, seed_heads, cfg.L, cfg.d, seed=cfg.seed)
    _REF.update(cfg=cfg, heads=[head_inputs_f64(q, k, v, 0, h) for h in range(seed_heads)],
                g=global_flags(cfg.L, cfg.global_idx), ex=ExtraIndex(cfg.L, cfg.extra_idx))


def _ref_task(args):
    """One worker's share of a reference step: the oracle (attention_rows, fp64) on R random rows of
    one head; returns (seconds, useful nnz)."""
    import numpy as np
    from oracle import attention_rows
    from oracle.mask import mask_row_cols
    seed, R = args
    cfg = _REF["cfg"]
    rng = np.random.default_rng(seed)
    Q, K, V = _REF["heads"][seed % len(_REF["heads"])]
    rows = rng.choice(cfg.L, R, replace=False)
    nnz = sum(mask_row_cols(int(r), cfg.L, cfg.window, _REF["g"], _REF["ex"]).size for r in rows)
    t0 = time.perf_counter()
    attention_rows(Q, K, V, rows, cfg.window, _REF["g"], _REF["ex"])
    return time.perf_counter() - t0, nnz


def run_reference(args):
    """--impl reference: the oracle (as it stands) on the host cores, one bounded sample per step:
    os.cpu_count() single-threaded worker processes each evaluate 32 random rows of one head
    (oracle.attention_rows, fp64); the step's wall clock is the pool's."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import multiprocessing as mp
    from workloads import get_config
    world = int(os.environ.get("WORLD_SIZE", "1"))
    name = resolve_workload(args, max(world, args.gpus))
    cfg = get_config(name)
    if args.head_dim:
        import dataclasses
        cfg = dataclasses.replace(cfg, d=args.head_dim)
    strong = cfg.name == "C5"
    lo, hi = shard_for_rank(cfg, max(world, args.gpus), 0, strong)
    cores = os.cpu_count() or 1
    R = 32
    with mp.get_context("spawn").Pool(cores, initializer=_ref_init, initargs=(name, args.head_dim, 2)) as pool:
        step_no = 0

        def step():
            nonlocal step_no
            tasks = [(step_no * cores + i, R) for i in range(cores)]
            step_no += 1
            t0 = time.perf_counter()
            res = pool.map(_ref_task, tasks, chunksize=1)
            return time.perf_counter() - t0, sum(n for _, n in res)

        for _ in range(args.warmup):
            step()
        tot_t, tot_nnz = 0.0, 0
        for _ in range(args.steps):
            t, n = step()
            tot_t += t
            tot_nnz += n
    value = 4.0 * tot_nnz * cfg.d / tot_t / 1e12
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot_t / args.steps,
        "higher_is_better": True, "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": workload_config(cfg, args.gpus, strong, hi - lo),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": f"oracle.attention_rows (fp64) on {R} random rows of one (b,h) head per worker, "
                                   f"{cores} single-threaded worker processes per step, {cfg.name}"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_iiswc_lica22_b200 as mg
    from workloads import get_config

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        if world == 1 and args.gpus > 1:
            raise SystemExit("--gpus N > 1 must be launched with torchrun (one process per GPU)")
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)

    cfg = get_config(resolve_workload(args, world))
    if args.head_dim:
        import dataclasses
        cfg = dataclasses.replace(cfg, d=args.head_dim)
    strong = cfg.name == "C5"
    lo, hi = shard_for_rank(cfg, world, rank, strong)
    b_local = hi - lo
    t_plan = time.perf_counter()
    plan = mg.Plan(cfg.L, cfg.H, cfg.d, cfg.window, cfg.global_idx, cfg.extra_idx,
                   strip_max_cols=args.strip_max_cols, fine_kernel=args.fine_kernel,
                   concurrency=args.concurrency, tau=args.tau, dense_chunk=args.dense_chunk, block=args.block)
    plan_build_ms = 1e3 * (time.perf_counter() - t_plan)   # host, once per pattern (before inference)
    info = plan.info()
    BH = b_local * cfg.H
    useful = 4.0 * info["nnz_total"] * cfg.d * BH                      # this rank
    useful_job = 4.0 * info["nnz_total"] * cfg.d * cfg.H * (cfg.B if strong else cfg.B * world)

    q, k, v = batch_inputs(cfg, lo, hi, rank, strong)
    host = [torch.from_numpy(x.view(np.int16)).view(torch.bfloat16) for x in (q, k, v)]
    Q, K, V = (h.to(dev) for h in host)
    O = torch.empty_like(Q)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    def fwd():
        mg.sparse_attention_fwd(plan, Q, K, V, O, stream)

    for _ in range(args.warmup):
        if not args.no_flush:
            flush.zero_()
        fwd()
    torch.cuda.synchronize()

    # Each step is timed by the library's own CUDA events on `stream`: one pair bracketing the
    # forward's kernels (plus one boundary event between the fine and the coarse kernel when both
    # run), the same pair that gives the per-kernel durations for the roofline. Extra per-step
    # event pairs around the call would each add a stream drain point (~2-3 us on B200).
    sampler = ClockSampler(nvml_index(local))
    plan.set_profiling(True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    for i in range(args.steps):
        if not args.no_flush:
            flush.zero_()
        fwd()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    sampler.stop()
    prof, per_call = plan.get_profile_calls()
    plan.set_profiling(False)
    assert prof["calls"] == args.steps
    t_ms = torch.tensor([prof["total_ms"], float(np.median(per_call)), float(np.min(per_call))],
                        dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t_ms, op=dist.ReduceOp.MAX)
    total_ms, med_ms, min_ms = (float(x) for x in t_ms.tolist())
    ms_per_step = total_ms / args.steps
    value = useful_job / (ms_per_step * 1e-3) / 1e12

    # ---------------- warm-L2 figure (no flush between steps; reported beside the flushed value)
    plan.set_profiling(True)
    for _ in range(min(args.steps, 100)):
        fwd()
    torch.cuda.synchronize()
    pw = plan.get_profile()
    plan.set_profiling(False)
    warm_ms = pw["total_ms"] / max(1, pw["calls"])

    # ---------------- e2e: host buffers through the C ABI (H2D + fwd + D2H every step)
    hq, hk, hv = (h.pin_memory() for h in host)
    hO = torch.empty_like(hq).pin_memory()
    n_e2e = max(1, min(args.e2e_steps, args.steps))
    for _ in range(2):
        mg.sparse_attention_fwd_host(plan, hq, hk, hv, hO, stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(n_e2e):
        mg.sparse_attention_fwd_host(plan, hq, hk, hv, hO, stream)
    e1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = torch.tensor([e0.elapsed_time(e1) / n_e2e], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(e2e_ms, op=dist.ReduceOp.MAX)
    e2e_value = useful_job / (float(e2e_ms.item()) * 1e-3) / 1e12
    nbytes = Q.numel() * 2

    # ---------------- N>1: NCCL all_gather of O, timed separately (not part of the fwd)
    gather_ms = None
    if world > 1:
        gather_output(O, cfg.B, strong)
        torch.cuda.synchronize()
        dist.barrier()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record(stream)
        for _ in range(5):
            gather_output(O, cfg.B, strong)
        g1.record(stream)
        torch.cuda.synchronize()
        gt = torch.tensor([g0.elapsed_time(g1) / 5], dtype=torch.float64, device=dev)
        dist.all_reduce(gt, op=dist.ReduceOp.MAX)
        gather_ms = float(gt.item())

    # ---------------- roofline of the dominant kernel (live, from the library's own events)
    peaks, peak_src = load_peaks()
    coarse_avg = prof["coarse_ms"] / max(1, prof["calls"])
    fine_avg = prof["fine_ms"] / max(1, prof["calls"])
    roof = roofline(cfg, info, BH, coarse_avg, fine_avg, peaks, peak_src, sampler.summary(), dev, args)

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "strong" if strong else "weak",
        "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
        "config": workload_config(cfg, world, strong, b_local),
        "fwd_ms": {"mean": ms_per_step, "median": med_ms, "min": min_ms, "steps": args.steps,
                   "timing": "library CUDA events on the launch stream, first to last kernel of each call; "
                             "max over ranks"},
        "useful_gflop_per_gpu": useful / 1e9,
        "fwd_ms_warm_l2": warm_ms,
        "plan_build_ms": plan_build_ms,
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": 3 * nbytes, "d2h_bytes_per_step": nbytes,
                "ms_per_step": float(e2e_ms.item()),
                "path": "mg_sparse_attention_fwd_host (pinned host Q/K/V/O, copies inside the timed region)"},
        "gpu_launches": int(args.steps * info["kernels_per_fwd"]),
        "kernels_per_fwd": info["kernels_per_fwd"],
        "roofline": roof,
        "clocks": sampler.summary(),
        "plan": {k_: info[k_] for k_ in ("n_tiles", "n_full_tiles", "nnz_total", "nnz_fine", "nnz_fine_strip",
                                          "nnz_fine_cuda", "n_items", "computed_scores")},
        "paper_context": "Multigrain reports 2.07x (Longformer) / 1.55x (QDS) end-to-end over Triton, FP16, "
                         "A100/RTX 3090 (PAPER.md P:12); no absolute numbers are published",
    }
    if gather_ms is not None:
        line["allgather_O_ms"] = gather_ms
    if args.ablation:
        line["staged_ablation"] = staged_ablation(mg, plan, Q, K, V, O, stream, flush, useful, ms_per_step, args)
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_oracle_pool(cfg, args.cpu_seconds)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def roofline(cfg, info, BH, coarse_avg, fine_avg, peaks, peak_src, clk, dev, args):
    import torch
    if coarse_avg >= fine_avg:
        coarse_nnz = info["nnz_coarse"] + info["nnz_fine_strip"] + info["n_global"] * cfg.L
        flops = 4.0 * coarse_nnz * cfg.d * BH
        achieved = flops / (coarse_avg * 1e-3) / 1e12
        peak = peaks["bf16_tflops"]
        roof = {"kernel": "coarse_pp_kernel (tcgen05 SDDMM + online SpSoftmax + SpMM)", "bound": "tensor",
                "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                "avg_launch_ms": coarse_avg, "algorithmic_per_launch": flops,
                "algorithmic_rule": "4*d flops per valid element it owns (coarse + strip + dense-row)",
                "peak_source": peak_src + " bf16 burst", "traffic": None}
        # the pipe that actually bounds this kernel: one MUFU ex2 per computed score (K1)
        mhz = clk.get("sm_mhz") or clk.get("sm_max_mhz")
        if mhz:
            sms = torch.cuda.get_device_properties(dev).multi_processor_count
            exps = float(info["computed_scores"]) * BH
            mufu_peak = 16.0 * sms * mhz * 1e6 / 1e12          # Tex2/s: 16 ex2 / clk / SM (measured)
            mufu_ach = exps / (coarse_avg * 1e-3) / 1e12
            roof["mufu"] = {"achieved": mufu_ach, "peak": mufu_peak, "unit": "Tex2/s",
                            "frac": mufu_ach / mufu_peak, "exps_per_launch": exps,
                            "peak_rule": "16 ex2/clk/SM (tools/microbench/mufu_mix.cu) x SMs x median SM clock; "
                                         "a share of the exponentials runs on the FMA pipe (MG_EXP_EMU), so frac "
                                         "can exceed what MUFU alone would allow"}
    else:
        nbytes_f = info["nnz_fine_cuda"] * BH * (2 * cfg.d * 2 + 4) + info["n_fine_rows"] * BH * (2 * cfg.d + 264)
        achieved = nbytes_f / (fine_avg * 1e-3) / 1e9
        peak = peaks["hbm_gbs"]
        kname = ("fine_mma_kernel (warp-level tensor-core CSR)" if args.fine_kernel == 0
                 else "fine_rows_kernel (CUDA-core CSR)")
        roof = {"kernel": kname, "bound": "hbm", "achieved": achieved, "peak": peak,
                "unit": "GB/s", "frac": achieved / peak, "avg_launch_ms": fine_avg,
                "algorithmic_per_launch": nbytes_f,
                "algorithmic_rule": "per nnz: K row + V row (2*d*2 B) + 4 B index; per row: Q read + partial write",
                "note": "the gathered K/V rows of a head (4 MB) are served by L2, so the algorithmic rate can exceed "
                        "the HBM peak the north_star measures against (frac > 1); `traffic` (ncu DRAM bytes) is "
                        "what reached HBM; see `l2` for the fraction of the L2 gather ceiling",
                "peak_source": peak_src, "traffic": None}
        # the level that actually serves the gathers: L2 (K2)
        l2_peak = L2_GATHER_GBS
        roof["l2"] = {"achieved": achieved, "peak": l2_peak, "unit": "GB/s", "frac": achieved / l2_peak,
                      "peak_rule": "measured L2->SM gather ceiling, 8 lanes per 128-B row, 16-B loads, no arithmetic "
                                   "(tools/microbench/gather_bw.cu, B200)"}
    tr_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tr_path):
        tr = json.load(open(tr_path)).get(cfg.name, {})
        key = "coarse" if roof["bound"] == "tensor" else "fine"
        if key in tr:
            roof["traffic"] = tr[key].get("dram_bytes_per_launch")
            roof["traffic_source"] = tr[key].get("source")
            if "lts_bytes_per_launch" in tr[key]:
                roof["l2_traffic"] = tr[key]["lts_bytes_per_launch"]
    return roof


def staged_ablation(mg, plan, Q, K, V, O, stream, flush, useful, ms_per_step, args):
    """The paper's dataflow (S and P materialised, SDDMM -> 3-sweep SpSoftmax -> SpMM kernels), same
    inputs, same L2 flush, CUDA events on the same stream; serial and multi-stream."""
    import torch
    out = {}
    for name, ms_kw in (("serial", dict(multi_stream=False)), ("multi_stream", dict(multi_stream=True))):
        Os = mg.sparse_attention_fwd_staged(plan, Q, K, V, None, stream, **ms_kw)
        for _ in range(3):
            mg.sparse_attention_fwd_staged(plan, Q, K, V, Os, stream, **ms_kw)
        n_ab = max(3, min(50, args.steps))
        ab = []
        for _ in range(n_ab):
            if not args.no_flush:
                flush.zero_()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            mg.sparse_attention_fwd_staged(plan, Q, K, V, Os, stream, **ms_kw)
            a1.record(stream)
            ab.append((a0, a1))
        torch.cuda.synchronize()
        st_ms = sum(a.elapsed_time(b) for a, b in ab) / n_ab
        diff = (Os.float() - O.float()).abs()
        out[name] = {"ms_per_step": st_ms, "tflops": useful / (st_ms * 1e-3) / 1e12,
                     "fused_speedup": st_ms / ms_per_step, "steps": n_ab, "max_abs_vs_fused": float(diff.max())}
    out["path"] = "mg_sparse_attention_fwd_staged (S, P in HBM; SDDMM / SpSoftmax / SpMM kernels)"
    return out


if __name__ == "__main__":
    sys.exit(main())
