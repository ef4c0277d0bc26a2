"""GPU parity of the NCHW layout adapters (f4): the NCHW / OIHW entry
points against the fp64 oracle (on the NHWC view of the same data), element by element under
the north-star bound, conv and deconv, several widths; the result equals the NHWC call's."""
import pytest
import torch

import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from tests.gpu_util import assert_parity, inputs

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("r", [2, 3, 5, 7, 9])
@pytest.mark.parametrize("kind", ["conv", "deconv"])
def test_nchw_adapter(kind, r):
    x, w = inputs(kind, 2, 13, 37, 16, 40, r, r)  # NHWC x; KRSC (conv) / CRSK (deconv) w
    p = r // 2
    xc = x.permute(0, 3, 1, 2).contiguous().cuda()           # NCHW
    if kind == "conv":
        wc = w.permute(0, 3, 1, 2).contiguous().cuda()        # KRSC -> OIHW [K][C][R][S]
        y = i2cw.conv2d_nchw(xc, wc, p, p)
        y_nhwc = i2cw.conv2d_nhwc(x.cuda(), w.cuda(), p, p)
        yr, b = oracle.conv2d_nhwc(x, w, p, p)
    else:
        wc = w.permute(0, 3, 1, 2).contiguous().cuda()        # CRSK -> [C][K][R][S]
        y = i2cw.deconv2d_nchw(xc, wc, p, p)
        y_nhwc = i2cw.deconv2d_nhwc(x.cuda(), w.cuda(), p, p)
        yr, b = oracle.deconv2d_nhwc(x, w, p, p)
    torch.cuda.synchronize()
    y_as_nhwc = y.permute(0, 2, 3, 1)
    assert_parity(y_as_nhwc, yr, b)
    assert torch.equal(y_as_nhwc, y_nhwc)  # same kernels on the same data


def test_nchw_matches_torch_conv2d():
    g = torch.Generator().manual_seed(3)
    x = torch.rand((3, 24, 20, 21), generator=g) * 2 - 1
    w = torch.rand((32, 24, 3, 3), generator=g) * 2 - 1
    y = i2cw.conv2d_nchw(x.cuda(), w.cuda(), 1, 1)
    yt = torch.nn.functional.conv2d(x.double(), w.double(), padding=1)
    bt = torch.nn.functional.conv2d(x.double().abs(), w.double().abs(), padding=1)
    torch.cuda.synchronize()
    assert float(((y.double().cpu() - yt).abs() / bt).max()) <= 1e-4
