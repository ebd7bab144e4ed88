timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for ub in 0 1 2 4; do DDT_UB=$ub timeout 300 python bench.py --no-extras --mode nccl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('cfg1 ub=$ub', d['value'], d['modes']['nccl'])"; done
DDT_GROUP_ALWAYS=1 timeout 300 python bench.py --no-extras --mode nccl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('cfg1 group', d['value'], d['modes']['nccl'])"
