#!/bin/bash
# Round-end style measurements: default bench line (as the driver runs it), the reference arm,
# every BASELINE config through bench.py, clocks. Usage (under gpurun): bash tools/final_round.sh TAG
export TAG=${1:-r02}; OUT=gpurun_out; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/nvsmi_$TAG.txt
python bench.py > $OUT/bench_cfg2_$TAG.json 2> $OUT/bench_cfg2_$TAG.err; tail -c 400 $OUT/bench_cfg2_$TAG.json; echo
python bench.py --steps 20 --warmup 3 > $OUT/bench_cfg2_k20_$TAG.json 2>> $OUT/bench_cfg2_$TAG.err
python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref_$TAG.json 2>&1; tail -c 300 $OUT/bench_ref_$TAG.json; echo
rm -f $OUT/bench_all_$TAG.jsonl
for c in cfg1 cfg2 cfg3-r2 cfg3-r3 cfg3-r4 cfg3-r5 cfg3-r6 cfg3-r7 cfg3-r8 cfg3-r9 cfg4-r5 cfg4-r7 cfg5a cfg5b-c64 cfg5b-c128 cfg5b-c256 cfg5b-c512; do
  python bench.py --config $c --no-cpu --no-e2e --no-sweep --no-peak --steps 30 --warmup 5 >> $OUT/bench_all_$TAG.jsonl 2>>$OUT/bench_all_$TAG.err
done
python - <<'PY'
import json
for l in open("gpurun_out/bench_all_TAGX.jsonl".replace("TAGX", __import__("os").environ.get("TAG","r02"))):
    d = json.loads(l); r = d["roofline"]
    print(d["config"]["name"], d["config"]["F(m,r)"], round(d["value"], 1), "TFLOPS kernel_us", round(r["kernel_ms"] * 1e3, 1),
          "frac", round(r["frac"], 3), "frac_default", round(r.get("frac_default_table", r["frac"]), 3), "star", round(d["star"]["value"], 1))
PY
