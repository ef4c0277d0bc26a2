# A/B of two library builds on one box (tools only): parity of the experiment build on the strip
# tests, then bench.py alternating the builds. Usage: bash tools/strip_ab.sh EXP_LIB [configs...]
EXP=${1:-exp/libi2cw_old.so}; shift
CFGS=${@:-cfg2 cfg4-r5}
I2CW_LIB_EXPERIMENT=$PWD/$EXP python -m pytest tests/test_gpu_strip.py -x -q 2>&1 | tail -3
for cfg in $CFGS; do
for r in 1 2; do
for L in paper_conf_icpp_zhangzxyw24_b200/libi2cw.so $EXP; do
I2CW_LIB_EXPERIMENT=$PWD/$L timeout 300 python bench.py --config $cfg --steps 20 --warmup 5 --no-cpu --no-e2e --no-sweep 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$cfg $L', d['value'], d['roofline']['frac'])"
done; done; done
