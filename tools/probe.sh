#!/bin/bash
# One GPU probe call: parity tests, cfg2 bench with / without CTA pairs, CTA-0 traces.
# Usage (under gpurun): bash tools/probe.sh TAG
TAG=${1:-p}; OUT=gpurun_out; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/nvsmi_$TAG.txt
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_$TAG.log 2>&1; tail -3 $OUT/pytest_$TAG.log
for p in 0 1; do
  for c in ${CFGS:-cfg2 cfg3-r3 cfg5b-c64 cfg3-r9}; do
    I2CW_PAIR=$p timeout 120 python bench.py --config $c --no-cpu --no-e2e --steps 30 --warmup 3 2>>$OUT/sweep_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('pair=$p $c', round(d['value'],1), 'TFLOPS frac', round(d['roofline']['frac'],3), 'kernel_us', round(d['roofline']['kernel_ms']*1000,1))"
  done
done | tee $OUT/sweep_$TAG.txt
for p in 0 1; do
  I2CW_PAIR=$p I2CW_LIB_EXPERIMENT=paper_conf_icpp_zhangzxyw24_b200/libi2cw_trace.so timeout 120 python tools/trace_run.py cfg2 > $OUT/trace_${TAG}_pair$p.txt 2>&1
  TIMELINE=1 TL_FROM=40000 I2CW_PAIR=$p I2CW_LIB_EXPERIMENT=paper_conf_icpp_zhangzxyw24_b200/libi2cw_trace.so timeout 120 python tools/trace_run.py cfg2 > $OUT/timeline_${TAG}_pair$p.txt 2>&1
done
grep -E "^WG|issuer0|math|in_full" $OUT/trace_${TAG}_pair*.txt
