#!/bin/bash
# Timing ablations of the fused kernel (results are wrong under I2CW_ABLATE; timing only).
# Needs a library built with make ABLATION=1 (the production build has no ablation branches).
# Usage (under gpurun): bash tools/ablate.sh TAG [configs...]
TAG=${1:-abl}; shift
CFGS=${@:-cfg2 cfg3-r3 cfg3-r7 cfg5b-c512}
OUT=gpurun_out; mkdir -p $OUT
for c in $CFGS; do
  for a in 0 1 2 4 8 16 5 3 7; do
    ms=$(I2CW_ABLATE=$a python bench.py --config $c --no-cpu --no-e2e --steps 30 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['kernel_ms']*1000,1))")
    echo "$c ablate=$a kernel_us=$ms"
  done
  ms=$(I2CW_PAIR=1 python bench.py --config $c --no-cpu --no-e2e --steps 30 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['roofline']['kernel_ms']*1000,1))")
  echo "$c pair kernel_us=$ms"
done | tee $OUT/ablate_$TAG.txt
