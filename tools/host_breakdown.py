"""Where a small call's host time goes: wall time per call, 300 calls back to back, for the
Python entry point and for the raw C-ABI calls underneath it. Usage: python tools/host_breakdown.py"""
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

import paper_conf_icpp_zhangzxyw24_b200 as i2cw  # noqa: E402


def per_call(f, n=300):
    for _ in range(20):
        f()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(n):
        f()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    return (t1 - t0) / n * 1e6, (t2 - t0) / n * 1e6


L = i2cw.lib()
for (N, H, W, C, K, r, p) in [(1, 56, 56, 64, 64, 3, 1), (1, 14, 14, 256, 256, 3, 1), (16, 56, 56, 64, 64, 3, 1)]:
    x = torch.rand((N, H, W, C), device="cuda")
    w = torch.rand((K, r, r, C), device="cuda")
    y = i2cw.conv2d_nhwc(x, w, p, p)
    u = i2cw.filter_transform(w)
    s = torch.cuda.current_stream().cuda_stream
    xp, wp, yp, up = x.data_ptr(), w.data_ptr(), y.data_ptr(), u.data_ptr()
    rows = [
        ("python conv2d_nhwc", lambda: i2cw.conv2d_nhwc(x, w, p, p)),
        ("python conv2d_nhwc out=", lambda: i2cw.conv2d_nhwc(x, w, p, p, out=y)),
        ("C i2cw_conv2d_nhwc", lambda: L.i2cw_conv2d_nhwc(N, H, W, C, K, r, r, p, p, xp, wp, yp, s)),
        ("C pretransformed", lambda: L.i2cw_conv2d_nhwc_pretransformed(N, H, W, C, K, r, r, p, p, xp, up, yp, s)),
        ("C filter_transform", lambda: L.i2cw_filter_transform(K, C, r, r, 0, wp, up, s)),
        ("C i2cw_version (ctypes floor)", lambda: L.i2cw_version()),
        ("torch.empty(y)", lambda: torch.empty(y.shape, device="cuda")),
        ("torch.cuda.current_stream()", lambda: torch.cuda.current_stream().cuda_stream),
    ]
    print(f"== N={N} {H}x{W} C=K={C} r={r}: host_us_per_call, incl_sync_us_per_call")
    for name, f in rows:
        h, t = per_call(f)
        print(f"{name:34s} {h:8.2f} {t:8.2f}", flush=True)
