timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for lib in default build/alt/libddt_smem.so default build/alt/libddt_smem.so; do
  if [ $lib != default ]; then export DDT_LIBDDT=$PWD/$lib; else unset DDT_LIBDDT; fi
  timeout 300 python bench.py --no-extras --mode nccl 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('cfg1 $lib', d['value'], d['modes']['nccl'])"
done
