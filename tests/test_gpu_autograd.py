"""Backward-data through autograd (paper_conf_icpp_zhangzxyw24_b200/autograd.py): the
gradient of conv(x, w, pad) w.r.t. x, produced by the deconvolution kernel, must match the
fp64 oracle's deconv(dy, w, pad) (the adjoint) within the parity bound,
and requesting dW must raise."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_icpp_zhangzxyw24_b200.autograd import conv2d, conv3d
from synthetic import make_w, make_x

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("r", [3, 5, 8])
def test_backward_data_matches_oracle(r):
    N, H, W, C, K, p = 2, 11, 19, 16, 24, r // 2
    x = make_x(0, N, H, W, C).cuda().requires_grad_(True)
    w = make_w(K, r, r, C).cuda()
    y = conv2d(x, w, p, p)
    dy = make_x(50, 50 + N, y.shape[1], y.shape[2], K)
    y.backward(dy.cuda())
    torch.cuda.synchronize()
    ref, bound = oracle.deconv2d_nhwc(dy, w.cpu(), p, p)
    got = x.grad.double().cpu().numpy()
    assert got.shape == ref.shape
    assert float(np.max(np.abs(got - ref) / np.maximum(bound, 1e-30))) <= 1e-4


def test_filter_gradient_not_offered():
    x = make_x(0, 1, 8, 8, 8).cuda()
    w = make_w(8, 3, 3, 8).cuda().requires_grad_(True)
    y = conv2d(x, w, 1, 1)
    with pytest.raises(NotImplementedError):
        y.sum().backward()


def test_backward_data_3d_matches_oracle():
    g = torch.Generator().manual_seed(5)
    x = (torch.rand((2, 6, 9, 13, 16), generator=g) * 2 - 1).cuda().requires_grad_(True)
    w = (torch.rand((24, 3, 3, 5, 16), generator=g) * 2 - 1).cuda()
    y = conv3d(x, w, 1, 1, 2)
    dy = torch.rand(y.shape, generator=g) * 2 - 1
    y.backward(dy.cuda())
    torch.cuda.synchronize()
    ref, bound = oracle.deconv3d_ndhwc(dy, w.cpu(), 1, 1, 2)
    got = x.grad.double().cpu().numpy()
    assert got.shape == ref.shape
    assert float(np.max(np.abs(got - ref) / np.maximum(bound, 1e-30))) <= 1e-4
