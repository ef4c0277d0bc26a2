"""Pins for the fp64 direct-conv oracle (oracle/direct_conv.c) — all -m "not gpu".

Each test pins the oracle to something other than itself: hand-worked values
(tests/golden/conv_hand.txt), torch's fp64 conv2d / conv_transpose2d (an
independent library), scipy.signal.correlate2d, exact-integer brute force,
delta inputs, the R=S=1 GEMM reduction, linearity, the deconv flip-transpose
and adjoint identities.
"""
import numpy as np
import pytest
import torch
import torch.nn.functional as F
from scipy.signal import correlate2d

import oracle
from synthetic import make_int_w, make_int_x, make_w, make_x
from tests.golden_io import load_sections


def torch_conv(x, w, ph, pw):
    # x NHWC, w KRSC -> NHWC via torch NCHW conv2d in fp64
    xt = torch.as_tensor(np.asarray(x, np.float64)).permute(0, 3, 1, 2)
    wt = torch.as_tensor(np.asarray(w, np.float64)).permute(0, 3, 1, 2)
    return F.conv2d(xt, wt, padding=(ph, pw)).permute(0, 2, 3, 1).numpy()


def torch_deconv(x, w, ph, pw):
    # w [C][R][S][K] -> conv_transpose2d weight [C_in=C][K][R][S]
    xt = torch.as_tensor(np.asarray(x, np.float64)).permute(0, 3, 1, 2)
    wt = torch.as_tensor(np.asarray(w, np.float64)).permute(0, 3, 1, 2)
    return F.conv_transpose2d(xt, wt, padding=(ph, pw)).permute(0, 2, 3, 1).numpy()


def test_hand_worked_conv_and_deconv():
    g = load_sections("conv_hand.txt")
    x = np.arange(1, 17, dtype=np.float32).reshape(1, 4, 4, 1)
    w = np.arange(1, 10, dtype=np.float32).reshape(1, 3, 3, 1)
    for pad in (0, 1):
        y, _ = oracle.conv2d_nhwc(x, w, pad, pad)
        exp = np.array(g[f"conv pad={pad}"], dtype=np.float64)
        np.testing.assert_array_equal(y[0, :, :, 0], exp)
        y, _ = oracle.deconv2d_nhwc(x, w, pad, pad)  # C=K=1: [C][R][S][K] == [1][3][3][1]
        exp = np.array(g[f"deconv pad={pad}"], dtype=np.float64)
        np.testing.assert_array_equal(y[0, :, :, 0], exp)


def test_all_ones_cfg1_corners_edges_interior():
    # cfg1 (N=1, 8x8, C=K=4, 3x3, pad 1) on all-ones: each output counts the in-range taps x C.
    x = np.ones((1, 8, 8, 4), np.float32)
    w = np.ones((4, 3, 3, 4), np.float32)
    y, b = oracle.conv2d_nhwc(x, w, 1, 1)
    assert y[0, 0, 0, 0] == 16 and y[0, 0, 7, 3] == 16 and y[0, 7, 7, 1] == 16
    assert y[0, 0, 3, 0] == 24 and y[0, 4, 0, 2] == 24
    assert np.all(y[0, 1:7, 1:7, :] == 36)
    np.testing.assert_array_equal(b, y)  # all positive: bound == value


@pytest.mark.parametrize("R,S,ph,pw", [(3, 3, 1, 1), (2, 5, 0, 2), (4, 3, 3, 1)])
def test_delta_input_and_delta_filter(R, S, ph, pw):
    H = W = 7
    x = np.zeros((1, H, W, 1), np.float32); x[0, 3, 2, 0] = 1
    w = np.zeros((1, R, S, 1), np.float32); w[0, R - 1, 0, 0] = 1
    y, _ = oracle.conv2d_nhwc(x, w, ph, pw)
    # y[p][q] = x[p-ph+R-1][q-pw+0]  -> single 1 at p = 3+ph-(R-1), q = 2+pw
    exp = np.zeros_like(y); p, q = 3 + ph - (R - 1), 2 + pw
    if 0 <= p < y.shape[1] and 0 <= q < y.shape[2]:
        exp[0, p, q, 0] = 1
    np.testing.assert_array_equal(y, exp)


def test_scipy_correlate2d_single_channel():
    rng = np.random.default_rng(0)
    x = rng.uniform(-1, 1, (1, 9, 11, 1)).astype(np.float32)
    w = rng.uniform(-1, 1, (1, 4, 3, 1)).astype(np.float32)
    for ph, pw in [(0, 0), (1, 2), (3, 1)]:
        y, _ = oracle.conv2d_nhwc(x, w, ph, pw)
        xp = np.pad(x[0, :, :, 0].astype(np.float64), ((ph, ph), (pw, pw)))
        exp = correlate2d(xp, w[0, :, :, 0].astype(np.float64), mode="valid")
        np.testing.assert_allclose(y[0, :, :, 0], exp, rtol=1e-13, atol=1e-13)


def test_r1s1_is_gemm():
    x = make_x(0, 2, 5, 6, 8).numpy()
    w = make_w(3, 1, 1, 8).numpy()
    y, _ = oracle.conv2d_nhwc(x, w, 0, 0)
    exp = x.reshape(-1, 8).astype(np.float64) @ w.reshape(3, 8).T.astype(np.float64)
    np.testing.assert_allclose(y.reshape(-1, 3), exp, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("R,S,ph,pw", [(3, 3, 1, 1), (2, 2, 1, 0), (4, 3, 0, 2), (1, 4, 2, 4)])
def test_brute_force_integers_exact(R, S, ph, pw):
    x = make_int_x(2, 5, 6, 3)
    w = make_int_w(2, R, S, 3)
    y, _ = oracle.conv2d_nhwc(x, w, ph, pw)
    yb = np.array(oracle.brute_conv_int(x.int().tolist(), w.int().tolist(), ph, pw), dtype=np.float64)
    np.testing.assert_array_equal(y, yb)
    wd = make_int_w(3, R, S, 2)  # [C=3][R][S][K=2]
    yd, _ = oracle.deconv2d_nhwc(x, wd, ph, pw)
    ydb = np.array(oracle.brute_deconv_int(x.int().tolist(), wd.int().tolist(), ph, pw), dtype=np.float64)
    np.testing.assert_array_equal(yd, ydb)


@pytest.mark.parametrize("R,S,ph,pw", [(3, 3, 1, 1), (5, 5, 2, 2), (7, 7, 3, 3), (2, 2, 1, 1), (4, 3, 0, 2), (9, 9, 4, 4)])
def test_torch_fp64_conv_and_bound(R, S, ph, pw):
    x = make_x(0, 2, 11, 10, 5).numpy()
    w = make_w(4, R, S, 5).numpy()
    y, b = oracle.conv2d_nhwc(x, w, ph, pw)
    np.testing.assert_allclose(y, torch_conv(x, w, ph, pw), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(b, torch_conv(np.abs(x), np.abs(w), ph, pw), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("R,S,ph,pw", [(3, 3, 1, 1), (5, 5, 2, 2), (7, 7, 3, 3), (2, 2, 1, 1), (4, 3, 0, 2), (3, 5, 2, 4)])
def test_torch_fp64_deconv_and_bound(R, S, ph, pw):
    x = make_x(0, 2, 9, 10, 5).numpy()
    w = make_w(5, R, S, 4).numpy()  # [C=5][R][S][K=4]
    y, b = oracle.deconv2d_nhwc(x, w, ph, pw)
    np.testing.assert_allclose(y, torch_deconv(x, w, ph, pw), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(b, torch_deconv(np.abs(x), np.abs(w), ph, pw), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("R,S,ph,pw", [(3, 3, 1, 1), (5, 5, 2, 2), (2, 2, 1, 1), (4, 3, 0, 2), (3, 5, 2, 4)])
def test_deconv_equals_conv_with_flipped_transposed_filter(R, S, ph, pw):
    # deconv(x, w, p) == conv(x, w', R-1-p) with w'[k][r][s][c] = w[c][R-1-r][S-1-s][k]
    # (negative padding = crop; SURVEY.md §8(c) reading 5)
    x = make_x(0, 1, 8, 9, 3).numpy()
    w = make_w(3, R, S, 4).numpy()  # [C=3][R][S][K=4]
    yd, _ = oracle.deconv2d_nhwc(x, w, ph, pw)
    wf = np.ascontiguousarray(w[:, ::-1, ::-1, :].transpose(3, 1, 2, 0))
    qh, qw = R - 1 - ph, S - 1 - pw
    if qh >= 0 and qw >= 0:
        yc, _ = oracle.conv2d_nhwc(x, wf, qh, qw)
    else:  # crop the input margin instead of negative padding
        xc = x[:, max(0, -qh): x.shape[1] - max(0, -qh), max(0, -qw): x.shape[2] - max(0, -qw), :]
        yc, _ = oracle.conv2d_nhwc(np.ascontiguousarray(xc), wf, max(qh, 0), max(qw, 0))
    np.testing.assert_allclose(yd, yc, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("R,S,ph,pw", [(3, 3, 1, 1), (5, 5, 2, 2), (4, 3, 0, 2)])
def test_adjoint_identity(R, S, ph, pw):
    # <conv(z, w), x> == <z, deconv(x, w)>  with w [K][R][S][C] read as the deconv's [C'][R][S][K']
    z = make_x(3, 4, 9, 8, 4).numpy()           # conv input  [1,9,8,C=4]
    w = make_w(5, R, S, 4).numpy()              # [K=5][R][S][C=4]
    yc, _ = oracle.conv2d_nhwc(z, w, ph, pw)     # [1,P,Q,5]
    x = make_x(7, 8, yc.shape[1], yc.shape[2], 5).numpy()
    yd, _ = oracle.deconv2d_nhwc(x, w, ph, pw)  # deconv filter [C'=5][R][S][K'=4]
    assert yd.shape == z.shape
    lhs = float(np.sum(yc * x.astype(np.float64)))
    rhs = float(np.sum(z.astype(np.float64) * yd))
    assert abs(lhs - rhs) <= 1e-10 * max(1.0, abs(lhs))


def test_linearity():
    x1 = make_x(0, 1, 7, 7, 4).numpy(); x2 = make_x(1, 2, 7, 7, 4).numpy()
    w = make_w(3, 3, 3, 4).numpy()
    y1, _ = oracle.conv2d_nhwc(x1, w, 1, 1); y2, _ = oracle.conv2d_nhwc(x2, w, 1, 1)
    y12, _ = oracle.conv2d_nhwc((2 * x1 - x2).astype(np.float32), w, 1, 1)
    np.testing.assert_allclose(y12, 2 * y1 - y2, rtol=1e-6, atol=1e-6)  # fp32 rounding of 2*x1-x2


def test_sampled_points_match_full():
    x = make_x(0, 2, 10, 9, 6).numpy(); w = make_w(5, 4, 3, 6).numpy()
    y, b = oracle.conv2d_nhwc(x, w, 2, 1)
    rng = np.random.default_rng(1)
    idx = np.stack([rng.integers(0, s, 50) for s in y.shape], 1)
    yp, bp = oracle.points("conv", x, w, 2, 1, idx)
    np.testing.assert_array_equal(yp, y[tuple(idx.T)]); np.testing.assert_array_equal(bp, b[tuple(idx.T)])
    wd = make_w(6, 3, 4, 5).numpy()
    y, b = oracle.deconv2d_nhwc(x, wd, 1, 2)
    idx = np.stack([rng.integers(0, s, 50) for s in y.shape], 1)
    yp, bp = oracle.points("deconv", x, wd, 1, 2, idx)
    np.testing.assert_array_equal(yp, y[tuple(idx.T)]); np.testing.assert_array_equal(bp, b[tuple(idx.T)])


def test_invalid_shape_raises():
    with pytest.raises(ValueError):
        oracle.conv2d_nhwc(np.zeros((1, 2, 2, 1), np.float32), np.zeros((1, 3, 3, 1), np.float32), 0, 0)
