#!/bin/bash
# Strip-kernel pipeline ablations (ABLATION build, results wrong): 2 no MMAs, 4 no epilogue,
# 8 no x TMA boxes, 16 no U loads; step time from the bench value.
LIB=$PWD/paper_conf_icpp_zhangzxyw24_b200/libi2cw_abl.so
for a in ${ABLS:-0 6 14 22 30 8 16 24}; do
  I2CW_ABLATE=$a I2CW_LIB_EXPERIMENT=$LIB timeout 120 python bench.py --config ${CFG:-cfg2} --no-cpu --no-e2e --no-sweep --no-peak --steps 30 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); fl=2*128*56*56*64*64*9; print('ablate=$a step_us', round(fl/d['value']/1e6,1))"
done
