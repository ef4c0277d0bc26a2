# Strip kernel ring depths (U slots, input stages, output buffers) after the warp-pair stores:
# step TFLOPS per I2CW_STRIP_DEPTHS setting (tools only). Usage (under gpurun): bash tools/strip_depths.sh
for cfg in ${CFGS:-cfg2 cfg5b-c128}; do
for r in 1 2; do
for d in 6,2,3 10,2,2 8,2,2 6,3,2 4,3,2 3,2,4; do
I2CW_STRIP_DEPTHS=$d timeout 200 python bench.py --config $cfg --steps 30 --warmup 5 --no-cpu --no-e2e --no-sweep --no-peak 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1])
import paper_conf_icpp_zhangzxyw24_b200 as i
print('$cfg', '$d', round(d['value'],1), 'TFLOPS frac', round(d['roofline']['frac'],3))"
done; done; done
