#!/bin/bash
# compute-sanitizer over small GPU configurations (run under gpurun): the fused
# kernels (all launch forms, variants, paired / spread plans) and the exchange
# kernel's protocols (ticket claims, LL words, per-chunk flags, fan-out, NCCL
# staging, captured graphs).
OUT=gpurun_out/sanitizer
mkdir -p $OUT
rm -f $OUT/summary.txt
K1="config1_vector or mixed_batch or shared_buffer or forms or direct_enqueue or halo_small or plan_replay or nan or grid_modes or segment_per_thread or pdl or enqueue_many or config3_sparse"
K2="mismatched or k_exchanges or float_layouts or nccl_mode or exchange_pairs"  # (kernels are serialised under the sanitizer: the SM-occupancy test cannot run there)
for tool in memcheck racecheck synccheck; do
  compute-sanitizer --tool $tool --error-exitcode 9 --target-processes all \
      python -m pytest tests/test_gpu_parity.py tests/test_gpu_halo.py -q -p no:cacheprovider -x -k "$K1" \
      > $OUT/$tool.log 2>&1
  echo "$tool (fused kernels) exit=$?" | tee -a $OUT/summary.txt
  grep -E "ERROR SUMMARY|passed|failed" $OUT/$tool.log | tail -3 | tee -a $OUT/summary.txt
  compute-sanitizer --tool $tool --error-exitcode 9 --target-processes all \
      python -m pytest tests/test_gpu_exchange_protocols.py -q -p no:cacheprovider -x -k "$K2" \
      > $OUT/${tool}_xchg.log 2>&1
  echo "$tool (exchange kernel) exit=$?" | tee -a $OUT/summary.txt
  grep -E "ERROR SUMMARY|passed|failed" $OUT/${tool}_xchg.log | tail -3 | tee -a $OUT/summary.txt
done
