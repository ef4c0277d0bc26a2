#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small cases of every kernel family:
# 2D conv + deconv (single CTA and CTA pair, alpha = 4 / 8 / 12, split tail), K-chunk launches,
# 3D conv + deconv, the NCHW adapters (transpose kernels) and the 1xTF32 mode.
# Usage (under gpurun): bash tools/sanitize.sh TAG   Outputs: gpurun_out/sanitizer_TAG_*.txt
TAG=${1:-r02}; mkdir -p gpurun_out
cat > /tmp/san.py <<'PY'
import torch, sys
sys.path.insert(0, '.')
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from synthetic import make_x, make_w
def run2(kind, N, H, W, C, K, R, S, ph, pw, **kw):
    x = make_x(0, N, H, W, C).cuda()
    w = (make_w(K, R, S, C) if kind == "conv" else make_w(C, R, S, K)).cuda()
    y = (i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc)(x, w, ph, pw, **kw)
    torch.cuda.synchronize()
    print(kind, tuple(y.shape), float(y.abs().sum()), kw)
for c in [("conv", 1, 8, 8, 4, 4, 3, 3, 1, 1), ("deconv", 2, 9, 13, 8, 12, 5, 5, 2, 2),
          ("conv", 3, 12, 20, 16, 40, 3, 3, 1, 1), ("conv", 2, 10, 14, 16, 40, 9, 9, 4, 4),
          ("conv", 2, 33, 41, 8, 40, 5, 5, 2, 2), ("deconv", 2, 33, 41, 8, 40, 5, 5, 2, 2),
          ("conv", 2, 9, 17, 16, 24, 3, 2, 1, 1), ("conv", 2, 9, 17, 256, 40, 3, 3, 1, 1)]:
    run2(*c)
run2("conv", 2, 9, 17, 16, 40, 3, 3, 1, 1, precision="1xtf32")
old = i2cw.debug_set_kchunk(6)  # K-chunk launches
run2("conv", 2, 9, 23, 40, 36, 3, 3, 1, 1)
i2cw.debug_set_kchunk(old)
x = torch.rand(1, 5, 6, 11, 16, device="cuda"); w = torch.rand(24, 3, 3, 3, 16, device="cuda")
print("conv3d", float(i2cw.conv3d_ndhwc(x, w, 1, 1, 1).abs().sum()))
w = torch.rand(16, 2, 3, 5, 12, device="cuda")
print("deconv3d", float(i2cw.deconv3d_ndhwc(x, w, 1, 1, 2).abs().sum()))
x = torch.rand(2, 16, 9, 13, device="cuda"); w = torch.rand(24, 16, 3, 3, device="cuda")
print("nchw", float(i2cw.conv2d_nchw(x, w, 1, 1).abs().sum()))
torch.cuda.synchronize()
PY
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python /tmp/san.py > gpurun_out/sanitizer_${TAG}_$tool.txt 2>&1; echo "$tool rc=$?"; tail -1 gpurun_out/sanitizer_${TAG}_$tool.txt
done
I2CW_PAIR=1 timeout 900 compute-sanitizer --tool memcheck python /tmp/san.py > gpurun_out/sanitizer_${TAG}_memcheck_pair.txt 2>&1; echo "pair memcheck rc=$?"; tail -1 gpurun_out/sanitizer_${TAG}_memcheck_pair.txt
