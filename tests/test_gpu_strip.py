"""GPU parity of the strip kernel (csrc/fused_strip.cuh): the planner's choice for
2D alpha = 8 problems whose images are tall enough that 32-lane strips waste few lanes.

Every output element is compared with the fp64 oracle under |err| <= 1e-4 sum|x||w|
(BASELINE.json north_star). The cases cover CTA pairs and single CTAs (the '*' path runs the
single-CTA form on a filter transformed in the base layout), runs of strips that straddle image
rows inside a unit (T_r not a multiple of 4), partial last row blocks, filter heights R = 1..7
(0..6 TMEM row shifts per chunk), deconvolution, C not a multiple of 8, K > 64 (two output-channel
blocks), concurrent K slices and K-chunked accumulation."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from tests.gpu_util import assert_parity, inputs, run_case

pytestmark = pytest.mark.gpu

CASES = [("conv", 2, 30, 40, 64, 64, 3, 3, 1, 1), ("conv", 3, 56, 30, 64, 64, 3, 3, 1, 1),
         ("deconv", 2, 28, 28, 64, 64, 5, 5, 2, 2), ("conv", 2, 29, 37, 64, 72, 3, 3, 1, 1),
         ("conv", 4, 28, 28, 128, 128, 3, 3, 1, 1), ("conv", 2, 28, 28, 40, 64, 3, 3, 1, 1),
         ("conv", 2, 57, 23, 64, 64, 3, 3, 1, 1), ("conv", 2, 28, 20, 64, 64, 1, 3, 0, 1),
         ("conv", 2, 28, 20, 64, 64, 2, 3, 1, 1), ("deconv", 2, 28, 28, 256, 256, 5, 5, 2, 2),
         ("conv", 1, 28, 28, 256, 256, 3, 3, 1, 1), ("conv", 2, 24, 31, 36, 64, 3, 3, 1, 1),
         ("conv", 2, 112, 40, 64, 64, 7, 7, 3, 3), ("conv", 2, 26, 26, 64, 64, 4, 4, 2, 2),
         ("conv", 2, 28, 28, 64, 64, 6, 6, 3, 3)]


@pytest.mark.parametrize("cfg", CASES, ids=lambda c: "_".join(map(str, c)))
def test_strip_every_element(cfg):
    kind, N, H, W, C, K, R, S, ph, pw = cfg
    p = i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)
    assert p["strip"] == 1, "the planner no longer picks the strip kernel for this shape"
    for lo, hi in ((-1.0, 1.0), (1.0, 2.0)):
        y, yr, b = run_case(kind, N, H, W, C, K, R, S, ph, pw, lo=lo, hi=hi)
        assert_parity(y, yr, b)


@pytest.mark.parametrize("cfg", [CASES[1], CASES[2], CASES[4]], ids=lambda c: "_".join(map(str, c)))
def test_strip_pair_and_single_cta_bitwise_equal(cfg):
    """The one-shot call runs the CTA-pair form; the pre-transformed call (U in the filter-only
    layout) the single-CTA form. Same summation order: bitwise-identical outputs, repeatable."""
    kind, N, H, W, C, K, R, S, ph, pw = cfg
    assert i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)["pair"] == 1
    x, w = inputs(kind, N, H, W, C, K, R, S)
    xd, wd = x.cuda(), w.cuda()
    f = i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc
    y1 = f(xd, wd, ph, pw)
    y1b = f(xd, wd, ph, pw)
    u = i2cw.filter_transform(wd, is_deconv=(kind == "deconv"))
    y2 = i2cw.conv2d_nhwc_pretransformed(xd, u, K, R, S, ph, pw, is_deconv=(kind == "deconv"))
    torch.cuda.synchronize()
    assert torch.equal(y1, y1b)
    assert torch.equal(y1, y2)


@pytest.mark.parametrize("kind", ["conv", "deconv"])
def test_strip_k_chunks(kind):
    """Long K loops as several launches (each from zero in TMEM, added by the TMA reduce-add)."""
    old = i2cw.debug_set_kchunk(6)
    try:
        cfg = (kind, 2, 28, 28, 40, 64, 3, 3, 1, 1)
        p = i2cw.debug_plan(*cfg)
        assert p["strip"] == 1 and p["NKC"] == 3
        y, yr, b = run_case(*cfg)
        assert_parity(y, yr, b)
    finally:
        i2cw.debug_set_kchunk(old)


def test_strip_pretransformed_layouts():
    """A pre-transformed U is in the filter-only plan's layout: the CTA-pair layout for C = 512 (long
    K loop), while a one-strip-group problem runs the single-CTA strip kernel in the one-shot call.
    The '*' call then runs the base kernel on the pair layout; both match the oracle."""
    cfg = ("conv", 1, 28, 20, 512, 64, 3, 3, 1, 1)
    kind, N, H, W, C, K, R, S, ph, pw = cfg
    p = i2cw.debug_plan(*cfg)
    assert p["strip"] == 1 and p["pair"] == 0
    x, w = inputs(kind, N, H, W, C, K, R, S)
    y1, yr, b = run_case(*cfg)
    u = i2cw.filter_transform(w.cuda())
    y2 = i2cw.conv2d_nhwc_pretransformed(x.cuda(), u, K, R, S, ph, pw)
    torch.cuda.synchronize()
    assert_parity(y1, yr, b)
    assert_parity(y2, yr, b)
