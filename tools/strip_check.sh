#!/bin/bash
# Strip kernel bring-up (under gpurun): GPU parity suite with the strip kernel forced wherever
# it applies, then the default planner; cfg sweep with the strip kernel on and off.
TAG=${1:-s}; OUT=gpurun_out; mkdir -p $OUT
I2CW_STRIP=1 timeout 600 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_strip1_$TAG.log 2>&1; tail -3 $OUT/pytest_strip1_$TAG.log
for S in 0 1; do
for c in ${CFGS:-cfg2 cfg5b-c64 cfg5b-c128 cfg3-r3}; do
  I2CW_STRIP=$S timeout 120 python bench.py --config $c --no-cpu --no-e2e --no-sweep --no-peak --steps 30 --warmup 3 2>>$OUT/sweep_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('strip=$S', '$c', round(d['value'],1), 'TFLOPS frac', round(d['roofline']['frac'],3), 'kernel_us', round(d['roofline']['kernel_ms']*1000,1))"
done
done | tee $OUT/sweep_$TAG.txt
