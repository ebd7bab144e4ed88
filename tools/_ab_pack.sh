#!/bin/bash
# A/B of alternative libraries on the dense-pack probe: tools/_ab_pack.sh lib1 lib2 ... ("default" = in-tree)
for lib in "$@"; do
  if [ "$lib" != default ]; then export DDT_LIBDDT=$PWD/$lib; else unset DDT_LIBDDT; fi
  r=$(PROBE_LIB_ARMS=0 timeout 300 python tools/pack_probe.py 5 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print([(c['S']>>20, c['plan']['alg_gbs'], c['plan_ub2']['alg_gbs']) for c in d['cells']])")
  c1=$(timeout 300 python bench.py --no-extras --mode nccl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['value'])")
  echo "$lib pack(S_MiB,plan,ub2)=$r cfg1_us=$c1"
done
