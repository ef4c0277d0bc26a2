#!/bin/bash
# One GPU session: tests, bench (headline + sweep), ncu launch list + one full capture.
# Usage (under gpurun): bash tools/gpu_round.sh TAG
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/nvsmi_$TAG.txt
python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu_$TAG.log 2>&1; tail -2 $OUT/pytest_gpu_$TAG.log
python bench.py > $OUT/bench_cfg2_$TAG.json 2> $OUT/bench_cfg2_$TAG.err; cat $OUT/bench_cfg2_$TAG.json; tail -3 $OUT/bench_cfg2_$TAG.err
python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref_$TAG.json 2>&1; cat $OUT/bench_ref_$TAG.json
rm -f $OUT/bench_sweep_$TAG.jsonl
for c in cfg1 cfg3-r2 cfg3-r3 cfg3-r4 cfg3-r5 cfg3-r6 cfg3-r7 cfg3-r8 cfg3-r9 cfg4-r5 cfg4-r7 cfg5a cfg5b-c64 cfg5b-c128 cfg5b-c256 cfg5b-c512; do
  python bench.py --config $c --no-cpu --no-e2e --steps 50 --warmup 5 >> $OUT/bench_sweep_$TAG.jsonl 2>>$OUT/bench_sweep_$TAG.err
done
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $OUT/launches_cfg2_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fused_tc -s 3 -c 1 -o $OUT/prof_cfg2_$TAG python bench.py --steps 1 --warmup 3 --no-cpu --no-e2e > $OUT/ncu_full_$TAG.log 2>&1
tail -1 $OUT/ncu_full_$TAG.log
