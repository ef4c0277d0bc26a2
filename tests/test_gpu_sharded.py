"""Batch-sharded verification over NCCL: each rank runs the fused kernel
on its contiguous shard of the global batch (per-image seeds: the data do not depend on the
sharding), sampled outputs are all_gathered over NCCL, and rank 0 checks them against the
fp64 oracle. Under pytest this is one rank on cuda:0 (a real NCCL process group of size 1);
the same file runs N ranks with
  torchrun --nproc-per-node N --master-addr 127.0.0.1 -m pytest tests/test_gpu_sharded.py -m gpu
The multi-rank host logic is covered on CPU by tests/test_shard_gloo.py (gloo, world 2)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from paper_conf_icpp_zhangzxyw24_b200.shard import gather_rows, max_over_ranks, sample_indices, shard_range
from synthetic import make_w, make_x

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("kind", ["conv", "deconv"])
def test_sharded_nccl_verification(kind):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    own = not dist.is_initialized()
    if own:
        if world == 1:
            os.environ["MASTER_ADDR"] = "127.0.0.1"
            os.environ["MASTER_PORT"] = str(_free_port())
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
    try:
        NG, H, W, C, K, r = 7, 20, 23, 64, 72, 3
        n0, n1 = shard_range(NG, world, rank)
        w = make_w(K, r, r, C) if kind == "conv" else make_w(C, r, r, K)
        x = make_x(n0, n1, H, W, C)
        f = i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record()
        y = f(x.to(dev), w.to(dev), 1, 1)
        ev1.record()
        torch.cuda.synchronize()
        t = max_over_ranks([ev0.elapsed_time(ev1)], device=dev)
        assert t[0] > 0
        idx = sample_indices(y.shape, 400, seed=3 + rank)
        vals = y[idx[:, 0].to(dev), idx[:, 1].to(dev), idx[:, 2].to(dev), idx[:, 3].to(dev)].double()
        rows = torch.cat([(idx + torch.tensor([[n0, 0, 0, 0]])).double().to(dev), vals[:, None]], 1)
        allrows = gather_rows(rows).cpu()
        if rank == 0:
            gi = allrows[:, :4].long().numpy()
            ref, bound = oracle.points(kind, make_x(0, NG, H, W, C), w, 1, 1, gi)
            err = np.abs(allrows[:, 4].numpy() - ref) / np.maximum(bound, 1e-30)
            assert allrows.shape[0] == 400 * world
            assert float(err.max()) <= 1e-4, f"max err/bound {err.max():.3e}"
    finally:
        if own:
            dist.destroy_process_group()
