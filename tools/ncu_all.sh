#!/bin/bash
# One ncu --set full capture of the fused kernel per BASELINE config (1 GPU) + the launch list
# of the cfg2 bench step. Usage (under gpurun): bash tools/ncu_all.sh TAG
TAG=${1:-r02}; OUT=gpurun_out; mkdir -p $OUT
for c in ${CFGS:-cfg2 cfg3-r2 cfg3-r3 cfg3-r4 cfg3-r5 cfg3-r6 cfg3-r7 cfg3-r8 cfg3-r9 cfg4-r5 cfg4-r7 cfg5a cfg5b-c64 cfg5b-c128 cfg5b-c256 cfg5b-c512}; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"fused_tc|fused_strip" -s 2 -c 1 -f \
      -o $OUT/ncu_${TAG}_$c python tools/ncu_one.py $c > $OUT/ncu_${TAG}_$c.log 2>&1
  echo "$c rc=$?"
  # summaries travel back; the reports do not (the returned gpurun_out/ is capped at 64 MiB),
  # except the headline config's
  python tools/ncu_summary.py $OUT/ncu_${TAG}_$c.ncu-rep $c $OUT/traffic_${TAG}.json > $OUT/ncu_${TAG}_${c}_summary.md 2>&1
  [ "$c" = "${KEEP:-cfg2}" ] || rm -f $OUT/ncu_${TAG}_$c.ncu-rep
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"fused|filter|zero|ksum" -c 24 --csv --log-file $OUT/launches_${TAG}_cfg2.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-sweep --no-peak > /dev/null 2>&1
echo "launch list rc=$?"
