#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small conv + deconv cases (both the
# single-CTA and the CTA-pair kernels). Usage (under gpurun): bash tools/sanitize.sh
# Outputs: gpurun_out/sanitizer_*.txt (committed copies: profiles/sanitizer/).
mkdir -p gpurun_out
cat > /tmp/san.py <<'PY'
import torch, sys
sys.path.insert(0, '.')
import paper_conf_icpp_zhangzxyw24_b200 as i2cw
from synthetic import make_x, make_w
for (kind, N, H, W, C, K, R, S, ph, pw) in [("conv", 1, 8, 8, 4, 4, 3, 3, 1, 1), ("deconv", 2, 9, 13, 8, 12, 5, 5, 2, 2), ("conv", 3, 12, 20, 16, 40, 3, 3, 1, 1), ("conv", 2, 10, 14, 16, 40, 9, 9, 4, 4), ("conv", 2, 33, 41, 8, 40, 5, 5, 2, 2), ("deconv", 2, 33, 41, 8, 40, 5, 5, 2, 2)]:
    x = make_x(0, N, H, W, C).cuda()
    w = (make_w(K, R, S, C) if kind == "conv" else make_w(C, R, S, K)).cuda()
    y = (i2cw.conv2d_nhwc if kind == "conv" else i2cw.deconv2d_nhwc)(x, w, ph, pw)
    torch.cuda.synchronize()
    print(kind, tuple(y.shape), float(y.abs().sum()))
PY
for tool in memcheck racecheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool python /tmp/san.py > gpurun_out/sanitizer_$tool.txt 2>&1; echo "$tool rc=$?"; tail -1 gpurun_out/sanitizer_$tool.txt
done
I2CW_PAIR=1 timeout 600 compute-sanitizer --tool memcheck python /tmp/san.py > gpurun_out/sanitizer_memcheck_pair.txt 2>&1; echo "pair memcheck rc=$?"; tail -1 gpurun_out/sanitizer_memcheck_pair.txt
