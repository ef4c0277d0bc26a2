"""Helpers for the -m gpu parity tests: run the CUDA path through the C ABI and compare
element by element with the fp64 oracle under the north-star bound
|y_gpu - y_oracle| <= TOL * sum|x||w|  (BASELINE.json north_star, TOL = 1e-4)."""
import numpy as np
import torch

import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from synthetic import make_w, make_x

TOL = 1e-4


def ratio(y_gpu, y_ref, bound):
    y = y_gpu.detach().cpu().double().numpy() if isinstance(y_gpu, torch.Tensor) else np.asarray(y_gpu, np.float64)
    assert y.shape == y_ref.shape, (y.shape, y_ref.shape)
    assert np.all(np.isfinite(y)), "non-finite output"
    err = np.abs(y - y_ref)
    # bound == 0 only where every term is 0: then the output must be exactly 0
    zero = bound == 0
    assert np.all(err[zero] == 0)
    return float(np.max(err[~zero] / bound[~zero])) if np.any(~zero) else 0.0


def assert_parity(y_gpu, y_ref, bound, tol=TOL):
    r = ratio(y_gpu, y_ref, bound)
    assert r <= tol, f"max |err| / sum|x||w| = {r:.3e} > {tol:.0e}"
    return r


def inputs(kind, N, H, W, C, K, R, S, lo=-1.0, hi=1.0, n0=0):
    x = make_x(n0, n0 + N, H, W, C, lo, hi)
    w = make_w(K, R, S, C, lo, hi) if kind == "conv" else make_w(C, R, S, K, lo, hi)
    return x, w


def run_case(kind, N, H, W, C, K, R, S, ph, pw, impl="tc", lo=-1.0, hi=1.0):
    x, w = inputs(kind, N, H, W, C, K, R, S, lo, hi)
    xd, wd = x.cuda(), w.cuda()
    if impl == "simt":
        y = i2cw.debug_conv_simt(xd, wd, ph, pw, is_deconv=(kind == "deconv"))
    elif kind == "conv":
        y = i2cw.conv2d_nhwc(xd, wd, ph, pw)
    else:
        y = i2cw.deconv2d_nhwc(xd, wd, ph, pw)
    torch.cuda.synchronize()
    f = oracle.conv2d_nhwc if kind == "conv" else oracle.deconv2d_nhwc
    y_ref, b = f(x, w, ph, pw)
    return y, y_ref, b
