# A/B of library builds on the configs[1] step (bench.py value, K = STEPS):
#   LIBS="default build/alt/libddt_x.so" [KNOB="DDT_NO_LEAN=1"] bash tools/_ab_libs.sh
cd ${GRAFT_REPO_ROOT:-.}
for rep in $(seq ${REPS:-2}); do
for L in ${LIBS:-default}; do
  l=$L; [ "$l" = "default" ] && l=""
  v=$(env DDT_LIBDDT=$l ${KNOB:-} timeout 300 python bench.py --no-extras --mode p2p --steps ${STEPS:-500} --warmup 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['value'], d['roofline']['latency_floor']['us'])")
  echo "[lib=$L ${KNOB:-}] cfg1_us floor_us = $v"
done; done
