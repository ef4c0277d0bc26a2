#!/bin/bash
# f1 measured selection: alpha 4 vs 8 (S = 2, 3) and alpha 16 vs default (S = 7..9), CTA pairs on/off.
OUT=gpurun_out; mkdir -p $OUT; TAG=${1:-vs}
run() {  # env... -- config
  python bench.py --config $1 --no-cpu --no-e2e --no-sweep --no-peak --steps 20 --warmup 3 2>>$OUT/vs_$TAG.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$1', '$ENVS', round(d['value'],1), 'TFLOPS kernel_us', round(r['kernel_ms']*1000,1), 'frac', round(r['frac'],3), 'frac_default', round(r.get('frac_default_table', r['frac']),3), d['config']['F(m,r)'])"
}
{
for c in cfg2 cfg3-r2 cfg3-r3 cfg5b-c64 cfg5b-c128 cfg5b-c256 cfg5b-c512; do
  for a in 8 4; do for p in 0 1; do ENVS="alpha=$a pair=$p"; I2CW_ALPHA=$a I2CW_PAIR=$p run $c; done; done
done
for c in cfg3-r7 cfg3-r8 cfg3-r9 cfg4-r7 cfg5a; do
  ENVS="default"; run $c
  ENVS="alpha16"; I2CW_ALPHA16=1 run $c
done
} | tee $OUT/vs_$TAG.txt
I2CW_ALPHA16=1 python tools/accuracy_table.py a16 > $OUT/acc_a16.log 2>&1; tail -22 $OUT/a16_accuracy_table.md
