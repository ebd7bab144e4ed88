#!/bin/bash
# A/B of environment knobs on the configs[1] step and the dense-pack probe:
#   tools/_ab_env.sh "" "DDT_NO_PDL=1" ...   ("" = defaults)
for knobs in "$@"; do
  c1=$(env $knobs timeout 300 python bench.py --no-extras --mode nccl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['value'], d['modes']['nccl']['isolated_flushed_us'])")
  r=$(env $knobs PROBE_LIB_ARMS=0 timeout 300 python tools/pack_probe.py 5 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print([(c['S']>>20, c['plan']['alg_gbs']) for c in d['cells']])")
  echo "[$knobs] cfg1_us(graph,isolated)=$c1 pack=$r"
done
