#!/bin/bash
# Strip-kernel timing ablations (ABLATION build; results wrong): kernel time per step from the
# bench's step value. Bits: 2 no MMAs/shifts, 4 no epilogue after the TMEM read, 32 no y writes.
LIB=$PWD/paper_conf_icpp_zhangzxyw24_b200/libi2cw_abl.so
for P in ${PAIRS:-1 0}; do for a in 0 32 4 2 6; do
  I2CW_STRIP_PAIR=$P I2CW_ABLATE=$a I2CW_LIB_EXPERIMENT=$LIB I2CW_STRIP=1 timeout 120 python bench.py --config ${CFG:-cfg2} --no-cpu --no-e2e --no-sweep --no-peak --steps 30 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); fl=2*128*56*56*64*64*9; print('pair=$P ablate=$a step_us', round(fl/d['value']/1e6,1))"
done; done
