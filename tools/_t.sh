timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for k in 0 1; do
DDT_NO_L2HINT=$k timeout 300 python tools/l2fetch_probe.py 2>&1 | grep '"set": 0' | head -2 | sed "s/^/nohint=$k /"
DDT_NO_L2HINT=$k PROBE_KNOBS='[{}]' timeout 600 python tools/comb_probe.py all x_any 2>&1 | grep class | sed "s/^/nohint=$k /"
DDT_NO_L2HINT=$k timeout 300 python bench.py --no-extras --mode nccl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('nohint=$k cfg1', d['value'])"
done
