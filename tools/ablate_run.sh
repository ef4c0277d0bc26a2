#!/bin/bash
# Timing ablations of the fused kernel (ablation build, results wrong): bash tools/ablate_run.sh TAG "0 32 512 ..."
# needs paper_conf_icpp_zhangzxyw24_b200/libi2cw_abl.so (make ABLATION=1 BUILD=build_abl LIB=libi2cw_abl.so)
TAG=$1; OUT=gpurun_out; mkdir -p $OUT
for c in ${CFGS:-cfg2}; do
  for a in $2; do
    I2CW_ABLATE=$a I2CW_LIB_EXPERIMENT=paper_conf_icpp_zhangzxyw24_b200/libi2cw_abl.so timeout 120 python bench.py --config $c --no-cpu --no-e2e --no-sweep --no-peak --steps 30 --warmup 3 2>>$OUT/abl_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c ablate=$a', 'kernel_us', round(d['roofline']['kernel_ms']*1000,1))"
  done
done | tee $OUT/abl_$TAG.txt
