#!/bin/bash
# Capture the round's ncu evidence on ONE GPU (run under gpurun from the repo root):
#   launch lists of the bench step (both exchange modes) and --set full captures
#   of the configs[1] step kernel, the configs[3] COMB kernel and a configs[4]
#   dense-pack kernel.  tools/summarize_profiles.py turns them into profiles/.
set -x
OUT=gpurun_out/prof_r
mkdir -p $OUT
for m in nccl p2p; do
  ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file $OUT/launches_cfg2_$m.csv \
      python bench.py --steps 100 --warmup 5 --no-extras --mode $m > /dev/null 2>&1
done
ncu --set full --clock-control none --import-source on -k regex:ddt_ -s 10 -c 1 -o $OUT/full_cfg2 \
    python bench.py --steps 12 --warmup 3 --no-extras --mode nccl > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:ddt_ -s 2 -c 1 -o $OUT/full_cfg4 \
    python tools/run_halo.py cfg4 nccl 4 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:ddt_ -s 2 -c 1 -o $OUT/full_cfg5 \
    python tools/run_pack.py 4194304 64 4 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:ddt_ -s 2 -c 1 -o $OUT/full_cfg3 \
    python tools/run_pack.py cfg3 32 4 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:ddt_ -s 2 -c 1 -o $OUT/full_cfg3cm \
    python tools/run_pack.py cfg3cm 32 4 > /dev/null 2>&1
ls -la $OUT
# summarise on the box (the five full reports exceed gpurun's 64 MiB return
# limit): raw pages + summaries come back, only the headline report is kept
python tools/summarize_profiles.py $OUT r01 gpurun_out/prof_sum > gpurun_out/prof_sum.log 2>&1
for r in $OUT/full_*.ncu-rep; do
  ncu -i $r --page raw --csv > ${r%.ncu-rep}_raw.csv 2>/dev/null
  ncu -i $r --page details --csv > ${r%.ncu-rep}_details.csv 2>/dev/null
done
ncu -i $OUT/full_cfg2.ncu-rep --page source --csv > $OUT/full_cfg2_source.csv 2>/dev/null
rm -f $OUT/full_cfg3.ncu-rep $OUT/full_cfg3cm.ncu-rep $OUT/full_cfg4.ncu-rep $OUT/full_cfg5.ncu-rep
du -sh $OUT gpurun_out
