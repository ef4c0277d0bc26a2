"""K-slice A/B on small grids (api.cu run_fused): device time of one call with the planner's
K slices vs forced off (debug_set_kslices(1)), per case. Usage: python tools/kslice_ab.py"""
import sys

sys.path.insert(0, ".")
import torch  # noqa: E402

import paper_conf_icpp_zhangzxyw24_b200 as i2cw  # noqa: E402

CASES = [("conv", 1, 14, 14, 256, 256, 3, 1), ("deconv", 2, 9, 23, 64, 36, 5, 2),
         ("conv", 1, 12, 20, 96, 64, 8, 4), ("deconv", 1, 9, 11, 256, 64, 5, 2), ("conv", 1, 10, 10, 256, 128, 7, 3),
         ("conv", 1, 28, 28, 128, 128, 3, 1), ("conv", 1, 28, 28, 256, 256, 5, 2),
         ("conv", 2, 14, 14, 512, 512, 3, 1), ("conv", 1, 56, 56, 64, 64, 3, 1),
         ("conv", 1, 7, 7, 512, 512, 3, 1), ("conv", 4, 14, 14, 256, 256, 3, 1),
         ("conv", 8, 56, 56, 128, 128, 3, 1), ("conv", 16, 56, 56, 64, 64, 3, 1)]


def time_us(f, reps=50):
    for _ in range(5):
        f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(reps):
        e0.record()
        f()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


print("case KSL items pair t_auto_us t_off_us speedup")
for c in CASES:
    kind, N, H, W, C, K, r, p = c
    g = torch.Generator(device="cuda").manual_seed(1)
    x = torch.rand((N, H, W, C), generator=g, device="cuda") * 2 - 1
    w = torch.rand((K, r, r, C) if kind == "conv" else (C, r, r, K), generator=g, device="cuda") * 2 - 1
    f = (lambda: i2cw.conv2d_nhwc(x, w, p, p)) if kind == "conv" else (lambda: i2cw.deconv2d_nhwc(x, w, p, p))
    pl = i2cw.debug_plan(kind, N, H, W, C, K, r, r, p, p)
    ta = time_us(f)
    ya = f()
    old = i2cw.debug_set_kslices(1)
    to = time_us(f)
    yo = f()
    i2cw.debug_set_kslices(old)
    torch.cuda.synchronize()
    d = float((ya - yo).abs().max())
    print(c, pl["KSL"], pl["NITEMS"], pl["pair"], f"{ta:.1f} {to:.1f} {to / ta:.2f} maxdiff={d:.2e}", flush=True)
