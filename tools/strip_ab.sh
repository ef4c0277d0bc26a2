python -m pytest tests/test_gpu_strip.py -x -q 2>&1 | tail -3
for cfg in cfg2 cfg4-r5; do
for r in 1 2; do
for L in exp/libi2cw_old.so paper_conf_icpp_zhangzxyw24_b200/libi2cw.so; do
I2CW_LIB_EXPERIMENT=$PWD/$L timeout 300 python bench.py --config $cfg --steps 20 --warmup 5 --no-cpu --no-e2e --no-sweep 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$cfg $L', d['value'], d['roofline']['frac'])"
done; done; done
