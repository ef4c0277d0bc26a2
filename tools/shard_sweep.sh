#!/bin/bash
# Per-GPU shard sizes of the batch split measured on one B200: each BASELINE
# config at N/G images for G = 1, 2, 4, 8 (per-image seeds, the same kernels a G-rank run
# launches on each rank). Projected strong scaling: G x (N/G images) / t(N/G).
OUT=gpurun_out; mkdir -p $OUT; TAG=${1:-sh}
python - <<'PY' | tee $OUT/shard_sweep_$TAG.txt
import os, sys, json
sys.path.insert(0, ".")
import torch, bench
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
dev = torch.device("cuda", 0)
flush = torch.empty(64 * 1024 * 1024, device=dev)
print("config G shard_images kernel+ft_us projected_job_TFLOPS efficiency_vs_G1")
for name in ["cfg2", "cfg3-r3", "cfg3-r7", "cfg3-r9", "cfg4-r7", "cfg5a", "cfg5b-c64", "cfg5b-c512"]:
    cfg = bench.CONFIGS[name]
    kind, N, H, W, C, K, R, S, ph, pw, _ = cfg
    P, Q = bench.out_hw(kind, H, W, R, S, ph, pw)
    g = torch.Generator(device=dev).manual_seed(7)
    w = torch.rand((K, R, S, C) if kind == "conv" else (C, R, S, K), generator=g, device=dev)
    f = i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc
    base = None
    for G in (1, 2, 4, 8):
        n = -(-N // G)  # the largest shard (shard_range gives the first N % G ranks one more)
        x = bench.make_x_device(0, n, H, W, C, dev)
        for _ in range(3):
            f(x, w, ph, pw)
        ts = []
        for _ in range(10):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); f(x, w, ph, pw); e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        t = sorted(ts)[len(ts) // 2]
        v = bench.direct_flops(cfg) / t / 1e12
        base = base or v
        print(name, G, n, round(t * 1e6, 1), round(v, 1), round(v / (G * base), 3), flush=True)
        del x
PY
