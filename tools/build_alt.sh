#!/bin/bash
# Build an alternative libddt.so with extra nvcc -D flags for kernel A/B
# experiments (the binding loads it via DDT_LIBDDT=<path>).
#   tools/build_alt.sh <name> -DDDT_V7_MINB=5 ...   -> build/alt/libddt_<name>.so
set -e
cd "$(dirname "$0")/.."
name=$1; shift
python paper_conf_cluster_chukzsp20_b200/build.py > /dev/null
mkdir -p build/alt
CS=paper_conf_cluster_chukzsp20_b200/csrc
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -std=c++17 -O3 -Xcompiler -fPIC \
  -I include -I /usr/local/cuda/include "$@" -c $CS/fused_kernel.cu -o build/alt/fused_$name.o
objs=$(ls build/libddt/*.o | grep -v fused_kernel)
/usr/local/cuda/bin/nvcc -shared -cudart static -gencode arch=compute_100a,code=sm_100a -o build/alt/libddt_$name.so \
  build/alt/fused_$name.o $objs -ldl -lpthread -lrt
echo build/alt/libddt_$name.so
