"""Strip-kernel bring-up: one small case under compute-sanitizer or plain, parity vs the oracle."""
import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import oracle
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from synthetic import make_x, make_w
cases = [("conv", 1, 40, 13, 64, 64, 3, 3, 1, 1), ("conv", 2, 9, 23, 40, 36, 3, 3, 1, 1),
         ("conv", 3, 56, 30, 64, 64, 3, 3, 1, 1), ("deconv", 2, 28, 28, 64, 64, 5, 5, 2, 2),
         ("conv", 16, 56, 56, 64, 64, 3, 3, 1, 1), ("conv", 3, 56, 30, 64, 64, 1, 3, 0, 1),
         ("conv", 3, 56, 30, 64, 64, 2, 3, 1, 1), ("conv", 3, 56, 30, 16, 64, 3, 3, 1, 1),
         ("conv", 1, 40, 13, 128, 64, 3, 3, 1, 1), ("conv", 1, 40, 13, 256, 64, 3, 3, 1, 1),
         ("conv", 3, 56, 30, 32, 64, 3, 3, 1, 1)]
which = [int(a) for a in sys.argv[1:]] or range(len(cases))
for ci in which:
    kind, N, H, W, C, K, R, S, ph, pw = cases[ci]
    x = make_x(0, N, H, W, C)
    w = make_w(K, R, S, C) if kind == "conv" else make_w(C, R, S, K)
    pl = i2cw.debug_plan(kind, N, H, W, C, K, R, S, ph, pw)
    y = (i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc)(x.cuda(), w.cuda(), ph, pw)
    torch.cuda.synchronize()
    yr, b = (oracle.conv2d_nhwc if kind == "conv" else oracle.deconv2d_nhwc)(x, w, ph, pw)
    yy = y.double().cpu().numpy()
    err = np.abs(yy - yr) / np.maximum(b, 1e-30)
    bad = np.argwhere(err > 1e-4)
    print(cases[ci], "strip", pl.get("strip"), "ROWS", pl["ROWS"], "PB", pl["PB"], "max err/B %.3e" % err.max(), "bad", len(bad))
    if len(bad):
        # which (p, q, k) are wrong
        ps = np.unique(bad[:, 1]); qs = np.unique(bad[:, 2]); ks = np.unique(bad[:, 3])
        print("  bad rows", ps[:40], "cols", qs[:40], "chans", ks[:20], "images", np.unique(bad[:, 0]))
        m = pl["m"]; rows = pl["ROWS"]
        from collections import Counter
        cnt = Counter((int(b[0]), int(b[1]) // rows, int(b[2]) // m) for b in bad)
        T_r = pl["T_r"]; PB = pl["PB"]
        by_strip = sorted(((n * PB + rb) * T_r + tw, c) for (n, rb, tw), c in cnt.items())
        print("  bad strips (index: count)", by_strip[:60])
        n, p, q, k = bad[0]
        print("  first bad", (n, p, q, k), yy[n, p, q, k], yr[n, p, q, k])

# regression of the error on per-(chunk, filter row) contributions (bring-up diagnostics)
if len(sys.argv) > 1 and sys.argv[1] == "2":
    kind, N, H, W, C, K, R, S, ph, pw = cases[2]
    x = make_x(0, N, H, W, C); w = make_w(K, R, S, C)
    y = i2cw.conv2d_nhwc(x.cuda(), w.cuda(), ph, pw); torch.cuda.synchronize()
    yr, b = oracle.conv2d_nhwc(x, w, ph, pw)
    err = (y.double().cpu().numpy() - yr)[1]  # image 1
    cols = []
    names = []
    for c in range(C // 8):
        for fh in range(R):
            wc = torch.zeros_like(w); wc[:, fh, :, 8 * c:8 * c + 8] = w[:, fh, :, 8 * c:8 * c + 8]
            yc, _ = oracle.conv2d_nhwc(x[1:2], wc, ph, pw)
            cols.append(yc[0].ravel()); names.append((c, fh))
    A = np.stack(cols, 1)
    coef, res, *_ = np.linalg.lstsq(A, err.ravel(), rcond=None)
    print("regression residual / |err|:", float(np.sqrt(np.sum((A @ coef - err.ravel()) ** 2)) / np.sqrt(np.sum(err ** 2))))
    print("coefs (chunk, fh): ", [(n, round(float(v), 3)) for n, v in zip(names, coef) if abs(v) > 0.02])
