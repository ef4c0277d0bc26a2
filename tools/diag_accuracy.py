"""Diagnostic (not a test): max err/bound and mean relative error of the tc path vs the
SIMT stepping stone on the same inputs, to attribute error to the contraction."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from tests.gpu_util import inputs

def stats(y, yr, b):
    y = y.double().cpu().numpy()
    e = np.abs(y - yr)
    return f"max err/B {np.max(e/b):.2e}  mean rel {np.mean(e/np.maximum(np.abs(yr),1e-30)):.2e}  mean err/B {np.mean(e/b):.2e}"

cases = [("conv", 2, 16, 32, 64, 64, 3, 3, 1, 1, 1.0, 2.0), ("conv", 2, 16, 32, 64, 64, 3, 3, 1, 1, -1.0, 1.0),
         ("conv", 2, 16, 32, 8, 8, 3, 3, 1, 1, 1.0, 2.0), ("conv", 2, 16, 32, 64, 64, 7, 7, 3, 3, 1.0, 2.0),
         ("conv", 2, 16, 32, 64, 64, 9, 9, 4, 4, -1.0, 1.0), ("conv", 2, 16, 32, 16, 16, 1 + 2, 3, 1, 1, -1.0, 1.0)]
for kind, N, H, W, C, K, R, S, ph, pw, lo, hi in cases:
    x, w = inputs(kind, N, H, W, C, K, R, S, lo, hi)
    xd, wd = x.cuda(), w.cuda()
    yt = i2cw.conv2d_nhwc(xd, wd, ph, pw)
    ys = i2cw.debug_conv_simt(xd, wd, ph, pw)
    torch.cuda.synchronize()
    yr, b = oracle.conv2d_nhwc(x, w, ph, pw)
    print(kind, N, H, W, C, K, R, S, (lo, hi))
    print("   tc  :", stats(yt, yr, b))
    print("   simt:", stats(ys, yr, b))

# full-size cfg2 sampled, printing details
kind, N, H, W, C, K, R, S, ph, pw = ("conv", 128, 56, 56, 64, 64, 3, 3, 1, 1)
g = torch.Generator(device="cuda").manual_seed(1234)
x = (torch.rand((N, H, W, C), generator=g, device="cuda") * 2 - 1).contiguous()
w = (torch.rand((K, R, S, C), generator=g, device="cuda") * 2 - 1).contiguous()
y = i2cw.conv2d_nhwc(x, w, ph, pw)
torch.cuda.synchronize()
print("finite", bool(torch.isfinite(y).all()))
for n in (0, 1, 64, 127):
    yr, b = oracle.conv2d_nhwc(x[n:n+1].cpu(), w.cpu(), ph, pw)
    e = np.abs(y[n:n+1].double().cpu().numpy() - yr) / b
    bad = np.argwhere(e > 1e-4)
    print("img", n, "max", e.max(), "nbad", len(bad), bad[:5].tolist())
