"""Batch sharding across GPUs -- host logic only, no arithmetic of the method.

Every output image y[n] depends only on x[n] and w (Table 1: the
convolution is independent per image), so the batch N is split into contiguous per-rank
ranges, one process per GPU, with NO collective on the timed path. torch.distributed
(NCCL on the GPU box, gloo in the CPU tests) is used only to

  * reduce timings with MAX over ranks (the job is as slow as its slowest rank), and
  * gather sampled outputs to rank 0 for verification against the oracle.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(n_global: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous [n0, n1) of the global batch for `rank`; the first n_global % world ranks
    take one image more (balanced, every image exactly once)."""
    if world < 1 or not 0 <= rank < world or n_global < 0:
        raise ValueError(f"bad shard request: n={n_global} world={world} rank={rank}")
    base, extra = divmod(n_global, world)
    n0 = rank * base + min(rank, extra)
    return n0, n0 + base + (1 if rank < extra else 0)


def max_over_ranks(values, device=None) -> list[float]:
    """Element-wise MAX of a list of floats over all ranks (identity without a process group)."""
    t = torch.tensor([float(v) for v in values], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        if dist.get_backend() == "gloo":  # gloo collectives on host tensors
            t = t.cpu()
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return t.tolist()


def gather_rows(local: torch.Tensor) -> torch.Tensor:
    """all_gather of per-rank [n_r, ...] tensors with possibly different n_r (padded to the
    largest, then trimmed); returns the concatenation in rank order on every rank."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return local
    if dist.get_backend() == "gloo" and local.is_cuda:  # gloo collectives on host tensors
        return gather_rows(local.cpu()).to(local.device)
    world = dist.get_world_size()
    n = torch.tensor([local.shape[0]], dtype=torch.int64, device=local.device)
    ns = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(ns, n)
    ns = [int(v.item()) for v in ns]
    nmax = max(ns)
    pad = torch.zeros((nmax,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    parts = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad)
    return torch.cat([p[:k] for p, k in zip(parts, ns)], 0)


def sample_indices(shape, npts: int, seed: int) -> torch.Tensor:
    """Deterministic (n, p, q, k) sample of an [N, P, Q, K] output, always including the last
    width column and the last channel (the in-kernel boundary tile and channel block)."""
    g = torch.Generator().manual_seed(seed)
    idx = torch.stack([torch.randint(0, int(s), (npts,), generator=g) for s in shape], 1)
    q = max(1, npts // 8)
    idx[:q, 2] = int(shape[2]) - 1
    idx[q:2 * q, 3] = int(shape[3]) - 1
    return idx
