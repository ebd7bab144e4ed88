#!/bin/bash
# Build and run the native scheduler-overhead harness (needs a GPU).
set -e
cd "$(dirname "$0")/.."
mkdir -p build
g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/sched_overhead.cpp -o build/sched_overhead \
    -L paper_conf_cluster_chukzsp20_b200 -l:libddt.so -Wl,-rpath,$(pwd)/paper_conf_cluster_chukzsp20_b200 \
    -L /usr/local/cuda/lib64 -lcudart
./build/sched_overhead
