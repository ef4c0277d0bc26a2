#!/bin/bash
# A/B of library builds: bash tools/ab.sh TAG lib1 lib2 ...   (libs under paper_conf_icpp_zhangzxyw24_b200/)
TAG=$1; shift; OUT=gpurun_out; mkdir -p $OUT
for rep in 1 2; do
for lib in "$@"; do
  for c in ${CFGS:-cfg2 cfg3-r3 cfg3-r9 cfg5b-c512}; do
    I2CW_LIB_EXPERIMENT=paper_conf_icpp_zhangzxyw24_b200/$lib timeout 120 python bench.py --config $c --no-cpu --no-e2e --no-sweep --no-peak --steps 30 --warmup 3 2>>$OUT/ab_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib $c', round(d['value'],1), 'TFLOPS frac', round(d['roofline']['frac'],3), 'kernel_us', round(d['roofline']['kernel_ms']*1000,1), 'star', round(d['star']['value'],1))"
  done
done
done | tee $OUT/ab_$TAG.txt
