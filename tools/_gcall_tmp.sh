for m in p2p nccl p2p; do timeout 300 python bench.py --steps 300 --warmup 10 --no-extras --mode $m 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); print('$m', d['value'], d['modes'])"; done
