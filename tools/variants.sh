#!/bin/bash
# Timing of experimental library builds (exp/lib_*.so) against the in-tree build.
# Usage (under gpurun): bash tools/variants.sh TAG "cfgs..." [ablate]
TAG=${1:-var}; CFGS=${2:-cfg2 cfg3-r3 cfg3-r7 cfg5b-c512}; AB=${3:-0}
OUT=gpurun_out; mkdir -p $OUT
for lib in base exp/lib_*.so; do
  for c in $CFGS; do
    if [ "$lib" = base ]; then unset I2CW_LIB_EXPERIMENT; else export I2CW_LIB_EXPERIMENT=$PWD/$lib; fi
    ms=$(I2CW_ABLATE=$AB timeout 300 python bench.py --config $c --no-cpu --no-e2e --steps 30 --warmup 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['roofline']['kernel_ms']*1000,1))")
    echo "$(basename $lib) $c ablate=$AB TFLOPS,kernel_us= $ms"
  done
done | tee -a $OUT/variants_$TAG.txt
