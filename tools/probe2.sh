#!/bin/bash
# GPU call: full parity suite (with prints), accuracy table, cfg2 trace, reduce->store ablation.
TAG=${1:-p2}; OUT=gpurun_out; mkdir -p $OUT
LIBDIR=paper_conf_icpp_zhangzxyw24_b200
timeout 1200 python -m pytest tests -m gpu -q -rA -s -p no:cacheprovider > $OUT/pytest_$TAG.log 2>&1; tail -3 $OUT/pytest_$TAG.log
timeout 900 python tools/accuracy_table.py $TAG > $OUT/acc_$TAG.log 2>&1; tail -2 $OUT/acc_$TAG.log
for p in 0; do
  I2CW_PAIR=$p I2CW_LIB_EXPERIMENT=$LIBDIR/libi2cw_trace.so timeout 120 python tools/trace_run.py cfg2 > $OUT/trace_${TAG}_pair$p.txt 2>&1
done
for a in 0 512 32 4; do
  I2CW_ABLATE=$a I2CW_LIB_EXPERIMENT=$LIBDIR/libi2cw_abl.so timeout 120 python bench.py --config cfg2 --no-cpu --no-e2e --steps 30 --warmup 3 2>>$OUT/abl_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('ablate=$a cfg2', round(d['value'],1), 'TFLOPS kernel_us', round(d['roofline']['kernel_ms']*1000,1))"
done | tee $OUT/abl_$TAG.txt
for c in cfg2 cfg3-r9 cfg5b-c512; do
  timeout 120 python bench.py --config $c --no-cpu --no-e2e --steps 30 --warmup 3 2>>$OUT/sweep_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['value'],1), 'TFLOPS frac', round(d['roofline']['frac'],3), 'kernel_us', round(d['roofline']['kernel_ms']*1000,1))"
done | tee $OUT/sweep_$TAG.txt
