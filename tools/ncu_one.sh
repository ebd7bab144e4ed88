#!/bin/bash
# One ncu --set full capture of the first ddt_ kernel after S skips:
#   tools/ncu_one.sh <name> <skip> <command...>   -> gpurun_out/ncu/<name>_{raw,details}.csv (+ .ncu-rep)
name=$1; skip=$2; shift 2
mkdir -p gpurun_out/ncu
ncu --set full --clock-control none --import-source on -k regex:ddt_ -s $skip -c 1 -f -o gpurun_out/ncu/$name "$@" > gpurun_out/ncu/$name.log 2>&1
ncu -i gpurun_out/ncu/$name.ncu-rep --page raw --csv > gpurun_out/ncu/${name}_raw.csv 2>/dev/null
ncu -i gpurun_out/ncu/$name.ncu-rep --page details --csv > gpurun_out/ncu/${name}_details.csv 2>/dev/null
