python -c "import __graft_entry__ as g; g.build()"
for lib in "" build/alt/libddt_r1.so "" build/alt/libddt_r1.so; do
  echo "== lib=$lib"
  DDT_LIBDDT=$lib timeout 600 python tools/pack_probe.py 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print([(c['S']>>20, c['plan']['alg_gbs'], c['copy']['alg_gbs']) for c in d['cells']])"
done
