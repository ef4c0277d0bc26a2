#!/bin/bash
# GPU tests + per-config step / fused-kernel / filter-transform times (under gpurun).
# Usage: bash tools/ft_sweep.sh TAG
TAG=${1:-ft}; OUT=gpurun_out; mkdir -p $OUT
python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_$TAG.log 2>&1; tail -2 $OUT/pytest_$TAG.log
for c in ${CFGS:-cfg2 cfg3-r3 cfg3-r5 cfg3-r7 cfg3-r9 cfg4-r7 cfg5b-c512}; do
  python bench.py --config $c --no-cpu --no-e2e --steps 30 --warmup 3 2>>$OUT/ft_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', round(d['value'],1), 'TFLOPS step_us', round(d['ms_per_step']*1000,1), 'kernel_us', round(r['kernel_ms']*1000,1), 'ft_us', round(r['filter_transform_ms']*1000,1))"
done | tee $OUT/ft_$TAG.txt
