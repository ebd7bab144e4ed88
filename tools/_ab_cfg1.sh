# A/B of environment knobs / library builds on the configs[1] step (bench.py value, K = 500):
#   KNOBS="x DDT_UB=2" LIB=build/alt/libddt_x.so bash tools/_ab_cfg1.sh   ("x" = defaults)
python -c "import __graft_entry__ as g; g.build()"
for knobs in ${KNOBS:-x "DDT_SPREAD_ALWAYS=1" "DDT_UB=2" "DDT_NO_PHASE=1" "DDT_GROUP_ALWAYS=1"}; do
  k=$knobs; [ "$k" = "x" ] && k=""
  v=$(env DDT_LIBDDT=${LIB:-} $k timeout 300 python bench.py --no-extras --mode p2p --steps ${STEPS:-500} --warmup 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['value'], d['roofline']['latency_floor']['us'])")
  echo "[lib=${LIB:-} $k steps=${STEPS:-500}] cfg1_us floor_us = $v"
done
