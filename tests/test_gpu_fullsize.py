"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py
times, on sampled outputs the oracle computes one by one (oracle.points)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from synthetic import make_w, make_x

pytestmark = pytest.mark.gpu

FULL = [("conv", 128, 56, 56, 64, 64, 3, 3, 1, 1)] + \
       [("conv", 64, 32, 32, 128, 128, r, r, r // 2, r // 2) for r in range(2, 10)] + \
       [("deconv", 64, 28, 28, 256, 256, 5, 5, 2, 2), ("deconv", 64, 28, 28, 256, 256, 7, 7, 3, 3),
        ("conv", 256, 112, 112, 64, 64, 7, 7, 3, 3)] + \
       [("conv", 256, 28, 28, c, c, 3, 3, 1, 1) for c in (64, 128, 256, 512)]


@pytest.mark.parametrize("cfg", FULL, ids=lambda c: "_".join(map(str, c)))
def test_full_size_sampled(cfg):
    kind, N, H, W, C, K, R, S, ph, pw = cfg
    g = torch.Generator(device="cuda").manual_seed(1234)
    x = (torch.rand((N, H, W, C), generator=g, device="cuda", dtype=torch.float32) * 2 - 1).contiguous()
    w = (torch.rand((K, R, S, C) if kind == "conv" else (C, R, S, K), generator=g, device="cuda", dtype=torch.float32) * 2 - 1).contiguous()
    y = (i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc)(x, w, ph, pw)
    torch.cuda.synchronize()
    assert bool(torch.isfinite(y).all())
    rng = np.random.default_rng(5)
    npts = 1500
    idx = np.stack([rng.integers(0, s, npts) for s in y.shape], 1)
    # always include the last width column (boundary tile), the last channel, the first and last
    # output rows (padding; the strip kernel's partial last row block) and the rows either side
    # of every strip row-block boundary (halo lanes of the next strip)
    idx[:100, 2] = y.shape[2] - 1
    idx[100:200, 3] = y.shape[3] - 1
    idx[200:300, 1] = y.shape[1] - 1
    idx[300:350, 1] = 0
    p = i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)
    edges = [e for rb in range(1, -(-y.shape[1] // p["ROWS"])) for e in (rb * p["ROWS"] - 1, rb * p["ROWS"])]
    if p["strip"] and edges:
        idx[350:550, 1] = np.asarray(edges)[rng.integers(0, len(edges), 200)]
    # only the images the sample touches go to the host
    imgs = np.unique(idx[:, 0])
    xs = x[torch.as_tensor(imgs, device="cuda")].cpu()
    remap = {int(n): i for i, n in enumerate(imgs)}
    idx_l = idx.copy()
    idx_l[:, 0] = [remap[int(n)] for n in idx[:, 0]]
    yr, b = oracle.points(kind, xs, w.cpu(), ph, pw, idx_l)
    yg = y[tuple(torch.as_tensor(idx.T, device="cuda"))].double().cpu().numpy()
    r = np.max(np.abs(yg - yr) / b)
    assert r <= 1e-4, r
