"""Multi-process (world_size 2, gloo, CPU) test of the batch-sharded N > 1 path
(paper_conf_icpp_zhangzxyw24_b200/shard.py): contiguous balanced shards,
MAX-over-ranks timing reduction, the uneven all_gather used for verification, and the
sampled-output verification bench.py --verify runs. Each rank computes its shard with the
fp64 oracle (no GPU here); the gathered batch must equal the unsharded oracle bit for bit
(per-image outputs do not depend on the sharding)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_icpp_zhangzxyw24_b200.shard import gather_rows, max_over_ranks, sample_indices, shard_range
from synthetic import make_w, make_x

N_GLOBAL, H, W, C, K = 5, 7, 9, 4, 8


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port):
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        n0, n1 = shard_range(N_GLOBAL, world, rank)
        w = make_w(K, 3, 3, C)
        y_local = torch.from_numpy(oracle.conv2d_nhwc(make_x(n0, n1, H, W, C), w, 1, 1, with_bound=False))
        y_all = gather_rows(y_local)
        t = max_over_ranks([float(rank), -float(rank)])
        assert t == [float(world - 1), 0.0]
        if rank == 0:
            full = oracle.conv2d_nhwc(make_x(0, N_GLOBAL, H, W, C), w, 1, 1, with_bound=False)
            assert y_all.shape == full.shape
            assert np.array_equal(y_all.numpy(), full)
        # sampled verification (bench.py --verify): gather (n, p, q, k, value) rows from every rank
        idx = sample_indices(y_local.shape, 64, seed=11 + rank)
        vals = y_local[idx[:, 0], idx[:, 1], idx[:, 2], idx[:, 3]]
        rows = torch.cat([idx.double() + torch.tensor([[n0, 0, 0, 0]], dtype=torch.float64), vals[:, None]], 1)
        allrows = gather_rows(rows)
        if rank == 0:
            gi = allrows[:, :4].long().numpy()
            ref, _ = oracle.points("conv", make_x(0, N_GLOBAL, H, W, C), w, 1, 1, gi)
            assert np.array_equal(allrows[:, 4].numpy(), ref)
            assert allrows.shape[0] == 64 * world
    finally:
        dist.destroy_process_group()


def _bench_worker(rank, world, port):
    """bench.py's strong-scaling split: each rank draws ITS images with bench.make_x_device
    (per-image seeds), the shards gathered over the process group equal the unsharded batch,
    and the MAX-over-ranks time reduction is what the whole-job value divides by."""
    import bench
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        n0, n1 = shard_range(N_GLOBAL, world, rank)
        xs = bench.make_x_device(n0, n1, H, W, C, torch.device("cpu"))
        x_all = gather_rows(xs)
        if rank == 0:
            assert torch.equal(x_all, bench.make_x_device(0, N_GLOBAL, H, W, C, torch.device("cpu")))
        t = max_over_ranks([0.5 + rank])
        assert t == [0.5 + world - 1]
        cfg = ("conv", N_GLOBAL, H, W, C, K, 3, 3, 1, 1, "")
        # whole-job throughput: all N_GLOBAL images over the slowest rank's time
        assert bench.direct_flops(cfg) == 2.0 * N_GLOBAL * H * W * C * K * 9
    finally:
        dist.destroy_process_group()


def test_bench_strong_scaling_split_gloo_world2():
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    mp.spawn(_bench_worker, args=(2, _free_port()), nprocs=2, join=True)


def test_shard_range_balanced_cover():
    for n in (0, 1, 5, 8, 13, 256):
        for world in (1, 2, 3, 4, 8):
            rs = [shard_range(n, world, r) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(rs, rs[1:]))
            sizes = [b - a for a, b in rs]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        shard_range(4, 2, 2)


def test_sharded_gather_gloo_world2():
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    mp.spawn(_worker, args=(2, _free_port()), nprocs=2, join=True)
