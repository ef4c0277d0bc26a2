"""Bring-up: x values the strip kernel's lane (sub 0, row 5) should see per chunk (compare with DUMP lines)."""
import sys
import torch
sys.path.insert(0, '.')
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from synthetic import make_x, make_w
N, H, W, C, K = 1, 40, 13, 64, 64
x = make_x(0, N, H, W, C)
# make x recognisable: value = 1000*row + 10*col + channel/8
for h in range(H):
    for w_ in range(W):
        for c in range(C):
            x[0, h, w_, c] = 1000 * h + 10 * w_ + c // 8
w = make_w(K, 3, 3, C)
y = i2cw.conv2d_nhwc(x.cuda(), w.cuda(), 1, 1)
torch.cuda.synchronize()
print(i2cw.debug_plan("conv", N, H, W, C, K, 3, 3, 1, 1))
