# A/B of environment knobs on the configs[1] step (bench.py value, K = STEPS):
#   KNOBS="x DDT_NO_LEAN=1" bash tools/_ab_env.sh     ("x" = defaults), REPS alternations
cd ${GRAFT_REPO_ROOT:-.}
for rep in $(seq ${REPS:-2}); do
for knobs in ${KNOBS:-x}; do
  k=$knobs; [ "$k" = "x" ] && k=""
  v=$(env $k timeout 300 python bench.py --no-extras --mode ${MODE:-p2p} --steps ${STEPS:-500} --warmup 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['value'], d['roofline']['latency_floor']['us'])")
  echo "[$k steps=${STEPS:-500}] cfg1_us floor_us = $v"
done; done
