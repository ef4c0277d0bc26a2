#!/bin/bash
# Ring-depth sweep (I2CW_DEPTHS=u,i,o: U k-steps, input stages, output staging buffers per warpgroup).
OUT=gpurun_out; mkdir -p $OUT; TAG=${1:-ds}
for c in ${CFGS:-cfg2 cfg3-r3 cfg3-r5 cfg3-r9 cfg5b-c64}; do
  for d in ${DEPTHS:-default 4,2,3 4,3,2 2,2,4 2,3,3 8,2,2}; do
    if [ "$d" = default ]; then unset I2CW_DEPTHS; else export I2CW_DEPTHS=$d; fi
    python bench.py --config $c --no-cpu --no-e2e --no-sweep --no-peak --steps 20 --warmup 3 2>>$OUT/ds_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', '$d', round(d['value'],1), 'TFLOPS kernel_us', round(d['roofline']['kernel_ms']*1000,1))"
  done
done | tee $OUT/ds_$TAG.txt
