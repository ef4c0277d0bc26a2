"""Split tail: the last units of the persistent schedule run as two one-pass
items that both reduce-add into y, which a zeroing kernel clears first; that kernel runs as a
programmatic dependent of the filter transform. These tests start from a y full of NaN or of a
previous result, in the two launch sequences the library uses (one-shot call, and
filter_transform + _pretransformed as bench.py times it), and require bitwise-identical results
that match the fp64 oracle on sampled outputs."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw

pytestmark = pytest.mark.gpu

# configs whose plan has a split tail (checked below): cfg2, cfg3 r = 7, and small ragged
# problems where every item is split
CASES = [("conv", 128, 56, 56, 64, 64, 3, 3, 1, 1), ("conv", 64, 32, 32, 128, 128, 7, 7, 3, 3),
         ("conv", 2, 33, 41, 8, 40, 5, 5, 2, 2), ("deconv", 2, 33, 41, 8, 40, 5, 5, 2, 2)]


def _sampled_ratio(kind, x, w, y, ph, pw, npts=600):
    rng = np.random.default_rng(11)
    idx = np.stack([rng.integers(0, s, npts) for s in y.shape], 1)
    idx[: npts // 2, 0] = np.maximum(0, y.shape[0] - 1 - rng.integers(0, 3, npts // 2))  # tail: last images
    imgs = np.unique(idx[:, 0])
    xs = x[torch.as_tensor(imgs, device="cuda")].cpu()
    remap = {int(n): i for i, n in enumerate(imgs)}
    idx_l = idx.copy()
    idx_l[:, 0] = [remap[int(n)] for n in idx[:, 0]]
    yr, b = oracle.points(kind, xs, w.cpu(), ph, pw, idx_l)
    yg = y[tuple(torch.as_tensor(idx.T, device="cuda"))].double().cpu().numpy()
    return float(np.max(np.abs(yg - yr) / b))


@pytest.mark.parametrize("cfg", CASES, ids=lambda c: "_".join(map(str, c)))
def test_split_tail_overwrites_stale_y(cfg):
    kind, N, H, W, C, K, R, S, ph, pw = cfg
    p = i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)
    if p["NITEMS"] == p["NFULL"]:
        pytest.skip("plan has no split tail")
    g = torch.Generator(device="cuda").manual_seed(99)
    x = torch.rand((N, H, W, C), generator=g, device="cuda") * 2 - 1
    w = torch.rand((K, R, S, C) if kind == "conv" else (C, R, S, K), generator=g, device="cuda") * 2 - 1
    is_deconv = kind == "deconv"
    P, Q = i2cw.out_shape(kind, N, H, W, K, R, S, ph, pw)[1:3]
    f = i2cw.deconv2d_nhwc if is_deconv else i2cw.conv2d_nhwc

    y1 = torch.full((N, P, Q, K), float("nan"), device="cuda")
    f(x, w, ph, pw, out=y1)
    torch.cuda.synchronize()
    assert bool(torch.isfinite(y1).all())

    # the bench sequence: filter transform, then the pretransformed call, into a y that holds
    # the previous result (a missing zeroing would double the tail)
    y2 = y1.clone()
    for _ in range(3):
        u = i2cw.filter_transform(w, is_deconv=is_deconv)
        i2cw.conv2d_nhwc_pretransformed(x, u, K, R, S, ph, pw, is_deconv=is_deconv, out=y2)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)

    assert _sampled_ratio(kind, x, w, y1, ph, pw) <= 1e-4
