python -c "import __graft_entry__ as g; g.build()"
for lib in ${LIBS:-"-"}; do
  [ "$lib" = "-" ] && lib=""
  echo "== lib=$lib"
  DDT_LIBDDT=$lib VARIANTS=${VARIANTS:-default} timeout 600 python tools/sparse_probe.py 32 2>&1 | tail -1
done
