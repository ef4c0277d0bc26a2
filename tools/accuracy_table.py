"""Accuracy table on B200 vs the fp64 oracle (writes profiles/<tag>_accuracy_table.md).

Rows mirror the paper's Table 3 (ofms shapes N x OH x OW x OC, C = K,
inputs U[1,2], "average relative error" vs an FP64 CPU convolution) at reduced batch N, plus
the r = 8, 9 (alpha = 12, R7) conv and deconv cases at C = K = 256 / 512 on both
U[-1,1] and U[1,2]. Every output element is compared; columns: max |err| / sum|x||w| (the
north-star bound is 1e-4) and the mean relative error (the paper's metric).
Usage (GPU box): python tools/accuracy_table.py TAG
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_icpp_zhangzxyw24_b200 as i2cw  # noqa: E402
from synthetic import make_w, make_x  # noqa: E402

# (r, paper's variant label, [(OH=OW, OC) rows of Table 3], paper mean rel err per row)
TABLE3 = [
    (2, "G8(7,2)", [(112, 64), (56, 128), (28, 256), (14, 512)], [1.43e-7, 2.01e-7, 2.90e-7, 4.31e-7]),
    (4, "G8(5,4)", [(80, 64), (40, 128), (20, 256), (10, 512)], [2.09e-7, 3.12e-7, 4.93e-7, 8.28e-7]),
    (3, "G8(6,3)", [(96, 64), (48, 128), (24, 256), (12, 512)], [2.04e-7, 2.69e-7, 3.68e-7, 5.20e-7]),
    (7, "G8(2,7)", [(128, 64), (64, 128), (32, 256), (16, 512)], [2.56e-7, 3.80e-7, 5.89e-7, 9.75e-7]),
    (5, "G8(4,5)", [(128, 64), (64, 128), (32, 256), (16, 512)], [2.10e-7, 3.05e-7, 4.57e-7, 7.21e-7]),
    (6, "G8(3,6)", [(96, 64), (48, 128), (24, 256), (12, 512)], [2.65e-7, 3.99e-7, 6.40e-7, 1.12e-6]),
    (8, "G16(9,8)", [(144, 64), (72, 128), (36, 256), (18, 512)], [9.86e-6, 1.04e-5, 1.18e-5, 1.48e-5]),
    (9, "G16(8,9)", [(128, 64), (64, 128), (32, 256), (16, 512)], [9.66e-6, 1.02e-5, 1.13e-5, 1.40e-5]),
]


def run(kind, N, OH, OW, C, K, r, lo, hi):
    p = r // 2
    if kind == "conv":
        H, W = OH - 2 * p + r - 1, OW - 2 * p + r - 1
    else:
        H, W = OH + 2 * p - r + 1, OW + 2 * p - r + 1
    x = make_x(0, N, H, W, C, lo, hi)
    w = make_w(K, r, r, C, lo, hi) if kind == "conv" else make_w(C, r, r, K, lo, hi)
    f = i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc
    y = f(x.cuda(), w.cuda(), p, p)
    torch.cuda.synchronize()
    yr, b = (oracle.conv2d_nhwc if kind == "conv" else oracle.deconv2d_nhwc)(x, w, p, p)
    yg = y.double().cpu().numpy()
    err = np.abs(yg - yr)
    nz = b > 0
    return float(np.max(err[nz] / b[nz])), float(np.mean(err[nz] / np.abs(yr[nz]))), \
        i2cw.debug_plan(kind, N, H, W, C, K, r, r, p, p)


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r02"
    lines = ["# Accuracy on B200 vs the fp64 oracle (" + tag + ")", "",
             "Every output element compared. `max err/B` = max |y - y_fp64| / sum|x||w| (north-star bound 1e-4);",
             "`mean rel` = mean |y - y_fp64| / |y_fp64| (the paper's Table 3 metric, PAPER.md:4187-4193).",
             "Reduced batch N (the error statistics are per element); C = K as in the paper.", "",
             "## Table 3 shapes, U[1,2] inputs (PAPER.md:4125-4185)", "",
             "| r | paper variant | ours F(m,r) alpha | N x OH x OW x OC | K-chunks | max err/B | mean rel | paper mean rel |",
             "|---|---|---|---|---|---|---|---|"]
    t0 = time.time()
    for r, lab, rows, paper in TABLE3:
        for (oh, oc), pm in zip(rows, paper):
            m, a, _ = i2cw.plan(r, oc)
            N = 1 if oh * oh * oc * oc * r * r > 2e9 else 2
            mx, mr, pl = run("conv", N, oh, oh, oc, oc, r, 1.0, 2.0)
            lines.append(f"| {r} | {lab} | F({m},{r}) {a} | {N}x{oh}x{oh}x{oc} | {pl['NKC']} | {mx:.2e} | {mr:.2e} | {pm:.2e} |")
            print(lines[-1], flush=True)
    lines += ["", "## alpha = 12 (r = 8, 9) at large C, conv and deconv, both input distributions", "",
              "| kind | r | C=K | inputs | N x OH x OW | K-chunks | max err/B | mean rel |", "|---|---|---|---|---|---|---|---|"]
    for kind in ("conv", "deconv"):
        for r in (8, 9):
            for c in (256, 512):
                for lo, hi in ((-1.0, 1.0), (1.0, 2.0)):
                    mx, mr, pl = run(kind, 2, 18, 18, c, c, r, lo, hi)
                    lines.append(f"| {kind} | {r} | {c} | U[{lo:g},{hi:g}] | 2x18x18 | {pl['NKC']} | {mx:.2e} | {mr:.2e} |")
                    print(lines[-1], flush=True)
    lines += ["", f"({time.time() - t0:.0f} s, oracle on {oracle.num_threads()} host threads)"]
    out = os.path.join(ROOT, "gpurun_out", f"{tag}_accuracy_table.md")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    open(out, "w").write("\n".join(lines) + "\n")
    print("wrote", out)


if __name__ == "__main__":
    main()
