python -c "import __graft_entry__ as g; g.build()"
for lib in "" build/alt/libddt_xminb6.so build/alt/libddt_xminb1.so; do
  echo "== lib=$lib"
  DDT_LIBDDT=$lib VARIANTS=direct,window,window_noll,window_xgrid1 ROUNDS=3 timeout 600 python tools/window_probe.py 2>&1 | tail -2
done
