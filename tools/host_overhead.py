"""Host overhead vs device time of one i2cw call on small problems.

  host_us   : wall time per call, 200 calls issued back to back (no sync)
  stream_us : device time per call over the same 200 back-to-back calls (events at the ends)
  single_us : events around ONE call after a sync (what a latency benchmark sees)
  graph_us  : one call captured in a CUDA graph, replayed (pure device time + graph launch)
Usage: python tools/host_overhead.py"""
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

import paper_conf_icpp_zhangzxyw24_b200 as i2cw  # noqa: E402

CASES = [("conv", 1, 14, 14, 256, 256, 3, 1), ("deconv", 2, 9, 23, 64, 36, 5, 2),
         ("conv", 1, 12, 20, 96, 64, 8, 4), ("deconv", 1, 9, 11, 256, 64, 5, 2), ("conv", 1, 10, 10, 256, 128, 7, 3),
         ("conv", 1, 56, 56, 64, 64, 3, 1), ("conv", 1, 7, 7, 512, 512, 3, 1),
         ("conv", 8, 56, 56, 128, 128, 3, 1), ("conv", 16, 56, 56, 64, 64, 3, 1),
         ("conv", 128, 56, 56, 64, 64, 3, 1)]


def ev():
    return torch.cuda.Event(enable_timing=True)


print("case KSL host_us stream_us single_us graph_us")
for c in CASES:
    kind, N, H, W, C, K, r, p = c
    g = torch.Generator(device="cuda").manual_seed(1)
    x = torch.rand((N, H, W, C), generator=g, device="cuda") * 2 - 1
    w = torch.rand((K, r, r, C) if kind == "conv" else (C, r, r, K), generator=g, device="cuda") * 2 - 1
    f = (lambda: i2cw.conv2d_nhwc(x, w, p, p)) if kind == "conv" else (lambda: i2cw.deconv2d_nhwc(x, w, p, p))
    for _ in range(10):
        f()
    torch.cuda.synchronize()
    n = 200
    e0, e1 = ev(), ev()
    t0 = time.perf_counter()
    e0.record()
    for _ in range(n):
        f()
    e1.record()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    host = (t1 - t0) / n * 1e6
    stream = e0.elapsed_time(e1) / n * 1e3
    singles = []
    for _ in range(30):
        torch.cuda.synchronize()
        a, b = ev(), ev()
        a.record()
        f()
        b.record()
        torch.cuda.synchronize()
        singles.append(a.elapsed_time(b) * 1e3)
    singles.sort()
    gus = float("nan")
    try:
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            f()
        torch.cuda.synchronize()
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr):
            f()
        gr.replay()
        torch.cuda.synchronize()
        a, b = ev(), ev()
        a.record()
        for _ in range(50):
            gr.replay()
        b.record()
        torch.cuda.synchronize()
        gus = a.elapsed_time(b) / 50 * 1e3
    except Exception as e:  # noqa: BLE001
        print("graph capture failed:", repr(e)[:200])
    pl = i2cw.debug_plan(kind, N, H, W, C, K, r, r, p, p)
    print(c, pl["KSL"], f"{host:.1f} {stream:.1f} {singles[len(singles) // 2]:.1f} {gus:.1f}", flush=True)
