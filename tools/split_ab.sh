#!/bin/bash
# A/B of the 3xTF32 split variants: speed (tools/ab.sh) and the U[1,2] mean error test.
OUT=gpurun_out; mkdir -p $OUT
for lib in libi2cw_s0.so libi2cw_s1.so libi2cw.so; do
  echo "== $lib"
  I2CW_LIB_EXPERIMENT=paper_conf_icpp_zhangzxyw24_b200/$lib python -m pytest tests/test_gpu_accuracy.py -k "mean_error_band or reduce_truncation" -q -s -p no:cacheprovider 2>&1 | grep -E "mean rel|passed|failed"
done | tee $OUT/split_errs.txt
