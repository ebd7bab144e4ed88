#!/bin/bash
# Round-2 ncu evidence on ONE GPU (run under gpurun from the repo root):
#   * the launch list of the bench command (gpu__time_duration per launch,
#     --clock-control none): the step kernel's share of the step;
#   * --set full captures of the configs[1] step kernel (DirectIPC), the
#     configs[1] window-protocol exchange kernel, COMB P=1, configs[2] sparse
#     B=32, and a configs[4] dense pack.
set -x
O=gpurun_out/r02
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_bench.csv \
    python bench.py --steps 100 --warmup 5 --no-extras --mode p2p > $O/launches_bench.out 2>&1
tools/ncu_one.sh cfg1_step 40 python bench.py --steps 30 --warmup 3 --no-extras --mode p2p
DDT_SELF_VIA_WINDOW=1 tools/ncu_one.sh cfg1_window 10 python tools/run_halo.py cfg2 p2p 12
tools/ncu_one.sh comb 2 python tools/run_halo.py cfg4 p2p 4
tools/ncu_one.sh sparse32 2 python tools/run_pack.py cfg3 32 4
tools/ncu_one.sh dense4m 2 python tools/run_pack.py 4194304 64 4
for f in gpurun_out/ncu/*.ncu-rep; do mv $f $O/ 2>/dev/null; done
mv gpurun_out/ncu/*_raw.csv gpurun_out/ncu/*_details.csv $O/ 2>/dev/null
rm -f $O/comb_nopair* $O/comb_pair*
ls -la $O
