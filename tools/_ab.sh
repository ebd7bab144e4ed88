#!/bin/bash
# scratch A/B over alternative libraries: tools/_ab.sh lib1 lib2 ... ("default" = in-tree)
for lib in "$@"; do
  if [ "$lib" != default ]; then export DDT_LIBDDT=$PWD/$lib; else unset DDT_LIBDDT; fi
  c1=$(timeout 300 python bench.py --no-extras --mode nccl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['value'])")
  c2=$(timeout 300 python tools/l2fetch_probe.py 2>&1 | grep '"set": 0' | head -1 | python -c "import json,sys; print(json.loads(sys.stdin.readline())['us'])")
  c2n=$(DDT_NO_NARROW=1 timeout 300 python tools/l2fetch_probe.py 2>&1 | grep '"set": 0' | head -1 | python -c "import json,sys; print(json.loads(sys.stdin.readline())['us'])")
  c3=$(PROBE_KNOBS='[{}]' PROBE_ROUNDS=5 timeout 600 python tools/comb_probe.py all 2>&1 | grep class | python -c "import json,sys; print(json.loads(sys.stdin.readline())['us'])")
  w=$(timeout 300 python tools/width_probe.py 2>&1 | grep -E 'pack16|direct8' | python -c "import json,sys; print([json.loads(l)['alg_GBs'] for l in sys.stdin])")
  echo "$lib cfg1_us=$c1 cfg2_us=$c2 cfg2_nonarrow_us=$c2n comb_us=$c3 pack16/direct8_GBs=$w"
done
