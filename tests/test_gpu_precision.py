"""GPU parity of the 1xTF32 precision mode (f4: "1xTF32 with looser
tolerance"): one tf32 product per Winograd point. Every output element against the fp64
oracle under the mode's stated bound |err| <= 4e-3 * sum|x||w| (include/i2cw.h, R17),
every filter width, conv and deconv, both input distributions; and a check that the mode is
really cheaper-but-coarser: its error exceeds the 3xTF32 error on the same inputs."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from tests.gpu_util import assert_parity, inputs, ratio

pytestmark = pytest.mark.gpu
TOL1 = i2cw.TOLERANCE["1xtf32"]


@pytest.mark.parametrize("r", list(range(2, 10)))
@pytest.mark.parametrize("kind", ["conv", "deconv"])
@pytest.mark.parametrize("dist", ["sym", "pos"])
def test_1xtf32_parity(kind, r, dist):
    lo, hi = (-1.0, 1.0) if dist == "sym" else (1.0, 2.0)
    x, w = inputs(kind, 2, 13, 37, 64, 40, r, r, lo, hi)
    p = r // 2
    f = i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc
    y1 = f(x.cuda(), w.cuda(), p, p, precision="1xtf32")
    y3 = f(x.cuda(), w.cuda(), p, p)
    torch.cuda.synchronize()
    yr, b = (oracle.conv2d_nhwc if kind == "conv" else oracle.deconv2d_nhwc)(x, w, p, p)
    e1 = assert_parity(y1, yr, b, tol=TOL1)
    e3 = ratio(y3, yr, b)
    print(f"{kind} r={r} {dist}: 1xTF32 max err/B {e1:.3e}, 3xTF32 {e3:.3e}")
    assert e1 > e3


def test_1xtf32_bad_precision_rejected():
    x, w = inputs("conv", 1, 8, 8, 8, 8, 3, 3)
    L = i2cw.lib()
    y = torch.empty((1, 8, 8, 8), device="cuda")
    rc = L.i2cw_conv2d_nhwc_prec(7, 0, 1, 8, 8, 8, 8, 3, 3, 1, 1, x.cuda().data_ptr(), w.cuda().data_ptr(),
                                 y.data_ptr(), None)
    assert rc == i2cw.I2CW_EINVAL
