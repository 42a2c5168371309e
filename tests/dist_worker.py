"""Worker for tests/test_dist_gloo.py, launched with torch.distributed.run (2 ranks, gloo, CPU).

Per rank: shard the batch (strong scaling) or draw its own seeded batch (weak scaling), run the
fp64 oracle as the stand-in forward, gather with the bench's gather helpers; rank 0 saves the
gathered arrays to argv[1].
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from oracle import dense_masked_attention, head_inputs_f64  # noqa: E402
from paper_conf_iiswc_lica22_b200.dist import gather_batches, gather_outputs, rank_seed, shard_range  # noqa: E402
from workloads import make_qkv  # noqa: E402

L, H, D, WINDOW, G = 64, 2, 64, 8, [0, 5]


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
    Bg = 5
    q, k, v = make_qkv(Bg, H, L, D, seed=3)
    lo, hi = shard_range(Bg, world, rank)
    full = gather_batches(torch.from_numpy(oracle_fwd(q[lo:hi], k[lo:hi], v[lo:hi])), Bg)
    qw, kw, vw = make_qkv(2, H, L, D, seed=rank_seed(0, rank))
    allw = gather_outputs(torch.from_numpy(oracle_fwd(qw, kw, vw)))
    if rank == 0:
        np.savez(sys.argv[1], full=full.numpy(), weak=allw.numpy())
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
