# configs[1] step (bench value, K = 500) and COMB / dense extras for library builds: LIBS="- alt.so ..."
python -c "import __graft_entry__ as g; g.build()"
for lib in ${LIBS:-"-"}; do
  [ "$lib" = "-" ] && lib=""
  v=$(DDT_LIBDDT=$lib timeout 300 python bench.py --no-extras --mode p2p --steps 500 --warmup 50 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['value'], d['roofline']['latency_floor']['us'])")
  echo "[lib=$lib] cfg1_us floor_us = $v"
done
