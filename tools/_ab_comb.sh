# COMB P = 1 A/B matrix (tools/comb_probe.py): knob sets x carveout, classes from $CLASSES
cd ${GRAFT_REPO_ROOT:-.}
K='[{}, {"DDT_GRID_MODE": "0"}, {"DDT_GRID_MODE": "1"}, {"DDT_NO_PAIR": "1"}, {"DDT_SPREAD": "0"}, {"DDT_NO_PDL": "1"}]'
for c in -1 0; do echo "carveout=$c"; DDT_CARVEOUT=$c PROBE_KNOBS="${KNOBS:-$K}" timeout 600 python tools/comb_probe.py ${CLASSES:-xface} 2>&1 | cut -c1-160; done
