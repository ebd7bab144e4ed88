timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
PROBE_KNOBS='[{}, {"DDT_SPREAD": "0"}, {"DDT_SPREAD": "0", "DDT_NO_GROUP": "1"}, {"DDT_UB": "2"}]' timeout 600 python tools/comb_probe.py all x_any dense 2>&1 | grep class
