#!/bin/bash
# A/B: phased units (default lib, V7 minB 4) vs DDT_NO_PHASE vs alt register budgets
export PROBE_KNOBS='[{}, {"DDT_NO_PHASE": "1"}]'
timeout 600 python -m pytest tests/test_gpu_phased.py -x -q 2>&1 | tail -3
for lib in default build/alt/libddt_m5.so build/alt/libddt_m3.so; do
  echo "== $lib"
  if [ $lib != default ]; then export DDT_LIBDDT=$PWD/$lib; fi
  timeout 400 python tools/comb_probe.py all dense 2>&1 | grep class
done
