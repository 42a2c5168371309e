"""World-size-2 gloo tests (CPU) of the scaling bench's host logic: batch sharding, per-rank seeding
and the output gather. The per-rank "forward" is the fp64 oracle on a tiny pattern, so the test
checks that sharded compute + gather equals the single-process result over the global batch.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

from paper_conf_iiswc_lica22_b200.dist import gather_batches, gather_outputs, rank_seed, shard_range


def test_shard_range_partitions():
    for B in (0, 1, 7, 8, 64):
        for world in (1, 2, 3, 8):
            spans = [shard_range(B, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == B
            assert all(spans[i][1] == spans[i + 1][0] for i in range(world - 1))
            assert max(h - l for l, h in spans) - min(h - l for l, h in spans) <= 1
    with pytest.raises(ValueError):
        shard_range(4, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_gloo_world2_shard_and_gather(tmp_path):
    """torch.distributed.run --nproc-per-node 2 (gloo): sharded oracle forward + gather equals the
    single-process result over the global batch; weak-scaling ranks draw distinct seeded batches."""
    import subprocess
    import sys
    from workloads import make_qkv
    sys.path.insert(0, os.path.dirname(__file__))
    import dist_worker as dw
    out = tmp_path / "gathered.npz"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}",
           os.path.join(os.path.dirname(__file__), "dist_worker.py"), str(out)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    res = np.load(out)
    q, k, v = make_qkv(5, dw.H, dw.L, dw.D, seed=3)
    assert np.array_equal(res["full"], dw.oracle_fwd(q, k, v))
    for rank in range(2):
        qw, kw, vw = make_qkv(2, dw.H, dw.L, dw.D, seed=rank_seed(0, rank))
        assert np.array_equal(res["weak"][rank], dw.oracle_fwd(qw, kw, vw))
