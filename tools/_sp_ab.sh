python -c "import __graft_entry__ as g; g.build()"
for lib in "" build/alt/libddt_segv16off.so; do
  echo "== lib=$lib"
  DDT_LIBDDT=$lib VARIANTS=default,rounds4,rounds1 timeout 600 python tools/sparse_probe.py 32 2>&1 | tail -1
  DDT_LIBDDT=$lib VARIANTS=default timeout 600 python tools/sparse_probe.py 16 2>&1 | tail -1
done
