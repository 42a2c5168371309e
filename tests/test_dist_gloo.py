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
    """torch.distributed.run --nproc-per-node 2 (gloo) over bench.py's own shard / input / gather
    functions: the sharded oracle forward + gather equals the single-process result over the global
    batch element for element (strong scaling, C5's scheme); weak-scaling ranks draw distinct batches."""
    import subprocess
    import sys
    sys.path.insert(0, os.path.dirname(__file__))
    import bench
    import dist_worker as dw
    out = tmp_path / "gathered.npz"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}",
           os.path.join(os.path.dirname(__file__), "dist_worker.py"), str(out)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    res = np.load(out)
    assert res["spans"].tolist() == [[0, 3], [3, 5]]
    q, k, v = bench.batch_inputs(dw.CFG, 0, dw.CFG.B, 0, strong=True)
    assert np.array_equal(res["full"], dw.oracle_fwd(q, k, v))
    for rank in range(2):
        qw, kw, vw = bench.batch_inputs(dw.CFG, 0, dw.CFG.B, rank, strong=False)
        assert np.array_equal(res["weak"][rank], dw.oracle_fwd(qw, kw, vw))
    assert not np.array_equal(res["weak"][0], res["weak"][1])


def test_bench_torchrun_world2_c5_line():
    """torchrun --nproc-per-node 2 bench.py --gpus 2 (the driver's N>1 launch) defaults to C5, the
    global batch of 64 sharded over the ranks: its reference arm runs on CPU (rank 0 prints one
    line, rank 1 exits 0) and carries scaling "strong" and the sharded config."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.join(root, "bench.py"),
           "--gpus", "2", "--impl", "reference", "--steps", "3", "--warmup", "3"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=root)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["scaling"] == "strong" and d["config"]["global_batch"] == 64 and d["config"]["B_per_gpu"] == 32
    assert d["config"]["workload"].startswith("C5")
