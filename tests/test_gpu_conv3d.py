"""GPU parity of the 3D path (f3: ND Im2col with the 1D Winograd Stage 2
unchanged) through the C ABI, element by element against the fp64 3D oracle under the
north-star bound |err| <= 1e-4 * sum|x||w|: every filter width S = 2..9, depth taps T = 1..3,
conv and deconv, ragged widths, several depth blocks per image, K <= 32 and K > 32 kernels,
K-chunked accumulation, and run-to-run determinism."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from tests.gpu_util import assert_parity

pytestmark = pytest.mark.gpu


def _rand(shape, seed, lo=-1.0, hi=1.0):
    g = torch.Generator().manual_seed(seed)
    return torch.rand(shape, generator=g, dtype=torch.float32) * (hi - lo) + lo


def run3(kind, N, D, H, W, C, K, T, R, S, pd, ph, pw, seed=0):
    x = _rand((N, D, H, W, C), 100 + seed)
    w = _rand((K, T, R, S, C) if kind == "conv" else (C, T, R, S, K), 200 + seed)
    f = i2cw.conv3d_ndhwc if kind == "conv" else i2cw.deconv3d_ndhwc
    y = f(x.cuda(), w.cuda(), pd, ph, pw)
    torch.cuda.synchronize()
    yr, b = (oracle.conv3d_ndhwc if kind == "conv" else oracle.deconv3d_ndhwc)(x, w, pd, ph, pw)
    return y, yr, b


@pytest.mark.parametrize("S", list(range(2, 10)))
@pytest.mark.parametrize("kind", ["conv", "deconv"])
def test_conv3d_every_width(kind, S):
    # 3x3xS-ish filter, same padding, W = 17 ragged against every m, K = 40 -> NT = 64
    y, yr, b = run3(kind, 2, 6, 7, 17, 16, 40, 3, 3, S, 1, 1, S // 2)
    assert_parity(y, yr, b)


@pytest.mark.parametrize("T,pd", [(1, 0), (2, 0), (2, 1), (3, 2)])
def test_conv3d_depth_taps_and_pads(T, pd):
    for kind in ("conv", "deconv"):
        y, yr, b = run3(kind, 1, 9, 6, 14, 8, 12, T, 2, 3, pd, 1, 1, seed=T)
        assert_parity(y, yr, b)


def test_conv3d_many_depth_blocks_and_channels():
    # OD = 20 output depths, small planes: several stacked-depth tile blocks per image
    y, yr, b = run3("conv", 2, 20, 5, 11, 72, 96, 3, 3, 3, 1, 1, 1, seed=5)
    assert_parity(y, yr, b)


def test_conv3d_k_chunked():
    old = i2cw.debug_set_kchunk(9)  # K loop of ceil(40/8) * T=3 * R=3 = 45 k-steps -> 5 chunks
    try:
        y, yr, b = run3("conv", 1, 5, 6, 13, 40, 24, 3, 3, 3, 1, 1, 1, seed=7)
        assert_parity(y, yr, b)
        y2, _, _ = run3("conv", 1, 5, 6, 13, 40, 24, 3, 3, 3, 1, 1, 1, seed=7)
        assert torch.equal(y, y2)
    finally:
        i2cw.debug_set_kchunk(old)


def test_conv3d_deterministic_and_2d_equivalence():
    x = _rand((2, 1, 10, 19, 16), 11)
    w = _rand((24, 1, 3, 5, 16), 12)
    y1 = i2cw.conv3d_ndhwc(x.cuda(), w.cuda(), 0, 1, 2)
    y2 = i2cw.conv3d_ndhwc(x.cuda(), w.cuda(), 0, 1, 2)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)
    # D = T = 1: the 3D call computes the 2D convolution (within the bound)
    y2d = i2cw.conv2d_nhwc(x[:, 0].cuda(), w[:, 0].cuda(), 1, 2)
    torch.cuda.synchronize()
    _, b = oracle.conv2d_nhwc(x[:, 0], w[:, 0], 1, 2)
    r = float(((y1[:, 0] - y2d).abs().double().cpu() / torch.as_tensor(b).clamp_min(1e-30)).max())
    assert r <= 2e-4


def test_conv3d_video_layer_full_check():
    """A video-style 3x3x3 layer (N=2, 8 frames of 28x28, C=K=64): every output element."""
    y, yr, b = run3("conv", 2, 8, 28, 28, 64, 64, 3, 3, 3, 1, 1, 1, seed=21)
    assert_parity(y, yr, b)
