python -c "import __graft_entry__ as g; g.build()"
for lib in ${LIBS:-"" build/alt/libddt_llsleep0.so build/alt/libddt_llsleep16.so}; do
  [ "$lib" = "-" ] && lib=""
  echo "== lib=$lib"
  DDT_LIBDDT=$lib VARIANTS=${VARIANTS:-direct,window} ROUNDS=3 timeout 600 python tools/window_probe.py ${WHICH:-all} 2>&1 | tail -2
done
