"""Pins of the 3D oracle (oracle/direct_conv3d.c: ND Im2col-Winograd equals
the direct ND convolution) against things other than itself: exact-integer brute force, the 2D
oracle (T = 1 and D = 1 reduce 3D to 2D exactly), torch conv3d / conv_transpose3d in fp64 (an
independent library), a closed-form all-ones case, delta inputs, and the deconv flip-transpose
and adjoint identities."""
import numpy as np
import pytest
import torch

import oracle
from synthetic import make_int_w, make_int_x


def _rand(shape, seed):
    g = torch.Generator().manual_seed(seed)
    return (torch.rand(shape, generator=g, dtype=torch.float32) * 2 - 1)


def test_conv3d_brute_force_integers():
    g = torch.Generator().manual_seed(3)
    x = torch.randint(-3, 4, (2, 4, 5, 6, 3), generator=g).float()
    w = torch.randint(-3, 4, (2, 3, 2, 3, 3), generator=g).float()
    for pads in ((0, 0, 0), (1, 1, 1), (2, 0, 1)):
        y, _ = oracle.conv3d_ndhwc(x, w, *pads)
        yb = oracle.brute_conv3d_int(x.numpy(), w.numpy(), *pads)
        assert np.array_equal(y, yb.astype(np.float64)), pads


def test_conv3d_t1_equals_2d_oracle():
    x = make_int_x(2, 6, 7, 4)
    w = make_int_w(3, 3, 3, 4)
    y3, b3 = oracle.conv3d_ndhwc(x[:, None], w[:, None], 0, 1, 1)
    y2, b2 = oracle.conv2d_nhwc(x, w, 1, 1)
    assert np.array_equal(y3[:, 0], y2) and np.array_equal(b3[:, 0], b2)
    yd3, _ = oracle.deconv3d_ndhwc(x[:, None], make_int_w(4, 3, 3, 3)[:, None], 0, 1, 1)
    yd2, _ = oracle.deconv2d_nhwc(x, make_int_w(4, 3, 3, 3), 1, 1)
    assert np.array_equal(yd3[:, 0], yd2)


@pytest.mark.parametrize("pads", [(0, 0, 0), (1, 1, 1), (2, 1, 0)])
def test_conv3d_matches_torch_fp64(pads):
    x, w = _rand((2, 5, 6, 7, 4), 1), _rand((3, 3, 2, 4, 4), 2)
    y, b = oracle.conv3d_ndhwc(x, w, *pads)
    yt = torch.nn.functional.conv3d(x.double().permute(0, 4, 1, 2, 3), w.double().permute(0, 4, 1, 2, 3),
                                    padding=pads).permute(0, 2, 3, 4, 1).numpy()
    assert np.max(np.abs(y - yt)) <= 1e-12 * max(1.0, np.max(b))


@pytest.mark.parametrize("pads", [(0, 0, 0), (1, 1, 1), (2, 1, 3)])
def test_deconv3d_matches_torch_fp64(pads):
    x, w = _rand((2, 4, 5, 6, 4), 3), _rand((4, 3, 2, 4, 5), 4)  # w [C][T][R][S][K]
    y, b = oracle.deconv3d_ndhwc(x, w, *pads)
    yt = torch.nn.functional.conv_transpose3d(x.double().permute(0, 4, 1, 2, 3), w.double().permute(0, 4, 1, 2, 3),
                                              padding=pads).permute(0, 2, 3, 4, 1).numpy()
    assert y.shape == yt.shape
    assert np.max(np.abs(y - yt)) <= 1e-12 * max(1.0, np.max(b))


def test_conv3d_all_ones_closed_form():
    # C = K = 1, 3x3x3 ones filter, pad 1: each output counts its in-range neighbours,
    # prod over axes of (2 at a border, 3 inside): corners 8, edges 12, faces 18, interior 27
    x = torch.ones((1, 4, 4, 4, 1))
    w = torch.ones((1, 3, 3, 3, 1))
    y, _ = oracle.conv3d_ndhwc(x, w, 1, 1, 1)
    cnt = np.array([2, 3, 3, 2])
    expect = cnt[:, None, None] * cnt[None, :, None] * cnt[None, None, :]
    assert np.array_equal(y[0, :, :, :, 0], expect.astype(np.float64))


def test_conv3d_delta():
    x = torch.zeros((1, 5, 5, 5, 2)); x[0, 2, 1, 3, 1] = 1.0
    w = torch.zeros((3, 2, 2, 2, 2)); w[2, 1, 0, 1, 1] = 1.0
    y, _ = oracle.conv3d_ndhwc(x, w, 0, 0, 0)
    nz = np.argwhere(y != 0)
    # y[d][p][q][k=2] = x[d+1][p+0][q+1][c=1]: the delta lands at (2-1, 1-0, 3-1)
    assert nz.tolist() == [[0, 1, 1, 2, 2]] and y[0, 1, 1, 2, 2] == 1.0


def test_deconv3d_flip_transpose_and_adjoint():
    x, w = _rand((1, 4, 5, 6, 3), 5), _rand((3, 3, 2, 3, 4), 6)  # w [C=3][T][R][S][K=4]
    pd, ph, pw = 1, 0, 2
    yd, _ = oracle.deconv3d_ndhwc(x, w, pd, ph, pw)
    wf = w.flip(1).flip(2).flip(3).permute(4, 1, 2, 3, 0).contiguous()  # [K][T][R][S][C]
    yc, _ = oracle.conv3d_ndhwc(x, wf, 3 - 1 - pd, 2 - 1 - ph, 3 - 1 - pw)
    assert np.max(np.abs(yd - yc)) <= 1e-12
    # adjoint: <conv(z, w^T-view), x> = <z, deconv(x, w)>, with the conv filter w' [C][T][R][S][K] read as
    # [K'=C][T][R][S][C'=K]
    z = _rand(yd.shape, 7)
    cz, _ = oracle.conv3d_ndhwc(z, w, pd, ph, pw)
    assert abs(float((cz * x.double().numpy()).sum()) - float((z.double().numpy() * yd).sum())) <= 1e-9
