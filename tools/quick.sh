#!/bin/bash
# Quick GPU iteration: parity tests, a bench sweep over the key configs, optional trace.
# Usage (under gpurun): bash tools/quick.sh TAG [trace]
TAG=${1:-q}; OUT=gpurun_out; mkdir -p $OUT
python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_$TAG.log 2>&1; tail -2 $OUT/pytest_$TAG.log
for c in ${CFGS:-cfg2 cfg3-r2 cfg3-r3 cfg3-r5 cfg3-r7 cfg3-r9 cfg4-r7 cfg5b-c64 cfg5b-c512}; do
  python bench.py --config $c --no-cpu --no-e2e --steps 30 --warmup 3 2>>$OUT/sweep_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['value'],1), 'TFLOPS frac', round(d['roofline']['frac'],3), 'kernel_us', round(d['roofline']['kernel_ms']*1000,1))"
done | tee $OUT/sweep_$TAG.txt
if [ "$2" = "trace" ]; then
  make -C paper_conf_icpp_zhangzxyw24_b200 TRACE=1 -j8 >/dev/null 2>&1 && python tools/trace_run.py cfg2 r3 > $OUT/trace_$TAG.txt 2>&1
  grep -E "^WG|issuer0|math|epilogue" $OUT/trace_$TAG.txt
fi
