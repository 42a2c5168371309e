"""Worker for tests/test_dist_gloo.py, launched with torch.distributed.run (2 ranks, gloo, CPU).

Drives bench.py's own multi-GPU host logic (shard_for_rank, batch_inputs, gather_output) with the
fp64 oracle as the stand-in forward: strong scaling (a global batch sharded in contiguous slices,
as for C5) and weak scaling (each rank its own seeded batch). Rank 0 saves the gathered arrays to
argv[1].
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import bench  # noqa: E402
from oracle import dense_masked_attention, head_inputs_f64  # noqa: E402
from workloads import Config  # noqa: E402

L, H, D, WINDOW = 64, 2, 64, 8
G = np.array([0, 5], np.int32)
CFG = Config("T5", 5, H, L, D, WINDOW, G, np.zeros((0, 2), np.int32), 3, "tiny strong-scaling batch")


def oracle_fwd(q, k, v):
    out = np.zeros(q.shape)
    for b in range(q.shape[0]):
        for h in range(q.shape[1]):
            Q, K, V = head_inputs_f64(q, k, v, b, h)
            out[b, h] = dense_masked_attention(Q, K, V, WINDOW, G, np.zeros((0, 2)))
    return out


def main():
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    lo, hi = bench.shard_for_rank(CFG, world, rank, strong=True)
    q, k, v = bench.batch_inputs(CFG, lo, hi, rank, strong=True)
    full = bench.gather_output(torch.from_numpy(oracle_fwd(q, k, v)), CFG.B, strong=True)
    lo, hi = bench.shard_for_rank(CFG, world, rank, strong=False)
    qw, kw, vw = bench.batch_inputs(CFG, lo, hi, rank, strong=False)
    allw = bench.gather_output(torch.from_numpy(oracle_fwd(qw, kw, vw)), CFG.B, strong=False)
    if rank == 0:
        np.savez(sys.argv[1], full=full.numpy(), weak=allw.numpy(), spans=np.array(
            [bench.shard_for_rank(CFG, world, r, strong=True) for r in range(world)]))
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
