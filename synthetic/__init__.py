"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no transforms, no convolution):
it only draws seeded random tensors with the shapes and value distributions of
the paper's workloads, so that both sides of a parity test see identical bytes.

Recipe:
  * x[n] ~ U[lo, hi) drawn per image from a generator seeded (1000 + n), where n
    is the GLOBAL image index, so a batch-sharded run sees the same data as an
    unsharded one.
  * w ~ U[lo, hi) seeded 7 (default).
  * default distribution U[-1, 1); the paper's accuracy experiment uses U[1, 2)
    (§6.2).
All tensors are fp32, contiguous, NHWC for feature maps and KRSC for filters
(Table 1).
"""
from __future__ import annotations

import torch

X_SEED_BASE = 1000
W_SEED = 7


def _uniform(shape, seed: int, lo: float, hi: float, device="cpu") -> torch.Tensor:
    g = torch.Generator(device=device)
    g.manual_seed(int(seed))
    t = torch.rand(shape, generator=g, dtype=torch.float32, device=device)
    return t.mul_(hi - lo).add_(lo)


def make_x(n0: int, n1: int, H: int, W: int, C: int, lo=-1.0, hi=1.0, device="cpu") -> torch.Tensor:
    """Images n0..n1-1 (global indices) of an NHWC fp32 feature map, one seed per image."""
    out = torch.empty((n1 - n0, H, W, C), dtype=torch.float32, device=device)
    for i, n in enumerate(range(n0, n1)):
        out[i] = _uniform((H, W, C), X_SEED_BASE + n, lo, hi, device)
    return out


def make_w(K: int, R: int, S: int, C: int, lo=-1.0, hi=1.0, seed=W_SEED, device="cpu") -> torch.Tensor:
    """A [K][R][S][C] fp32 filter (KRSC). For a deconvolution the same call with
    (K, C) swapped gives the [C][R][S][K] filter the deconv consumes."""
    return _uniform((K, R, S, C), seed, lo, hi, device)


def make_int_x(N, H, W, C, seed=11, lo=-3, hi=4):
    """Small-integer NHWC input (exact in fp32 and fp64) for brute-force pins."""
    g = torch.Generator().manual_seed(seed)
    return torch.randint(lo, hi, (N, H, W, C), generator=g).to(torch.float32)


def make_int_w(K, R, S, C, seed=13, lo=-3, hi=4):
    g = torch.Generator().manual_seed(seed)
    return torch.randint(lo, hi, (K, R, S, C), generator=g).to(torch.float32)
