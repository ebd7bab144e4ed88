#!/bin/bash
# compute-sanitizer over small GPU configurations (run under gpurun).
OUT=gpurun_out/sanitizer
mkdir -p $OUT
for tool in memcheck racecheck synccheck; do
  compute-sanitizer --tool $tool --error-exitcode 9 --target-processes all \
      python -m pytest tests/test_gpu_parity.py tests/test_gpu_halo.py -q -p no:cacheprovider -x \
      -k "config1_vector or mixed_batch or forms or direct_enqueue or halo_small or plan_replay or nan or grid_modes or segment_per_thread or pdl or enqueue_many or config3_sparse" \
      > $OUT/$tool.log 2>&1
  echo "$tool exit=$?" | tee -a $OUT/summary.txt
  grep -E "ERROR SUMMARY|passed|failed" $OUT/$tool.log | tail -3 | tee -a $OUT/summary.txt
done
