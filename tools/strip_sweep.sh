#!/bin/bash
# Strip kernel vs base kernel on every BASELINE config it can run (step TFLOPS, one B200).
OUT=gpurun_out; TAG=${1:-ss}
run() { timeout 180 python bench.py --config $1 --no-cpu --no-e2e --no-sweep --no-peak --steps 30 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$2 $1', round(d['value'],1), 'TFLOPS', d['config'].get('F(m,r)',''))"; }
for c in ${CFGS:-cfg2 cfg3-r3 cfg3-r4 cfg3-r5 cfg3-r6 cfg3-r7 cfg4-r5 cfg4-r7 cfg5a cfg5b-c64 cfg5b-c128 cfg5b-c256 cfg5b-c512}; do
  I2CW_STRIP=0 run $c base
  I2CW_STRIP=1 run $c strip
done | tee $OUT/strip_sweep_$TAG.txt
for c in cfg5b-c256 cfg5b-c512 cfg3-r3; do I2CW_ALPHA=8 I2CW_STRIP=1 run $c strip-a8; I2CW_ALPHA=8 I2CW_STRIP=0 run $c base-a8; done | tee -a $OUT/strip_sweep_$TAG.txt
