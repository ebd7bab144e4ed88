# COMB P = 1: library builds (LIBS) x knob sets (KNOBS), classes CLASSES (tools/comb_probe.py)
cd ${GRAFT_REPO_ROOT:-.}
if [ -z "$KNOBS" ]; then KNOBS='[{}]'; fi
for L in ${LIBS:-default}; do l=$L; [ "$l" = default ] && l=; echo "lib=$L"
  DDT_LIBDDT=$l PROBE_KNOBS="$KNOBS" timeout 600 python tools/comb_probe.py ${CLASSES:-xface all} 2>&1 | sed 's/"msgs.*"us"/ us/; s/, "min_us.*//'
done
