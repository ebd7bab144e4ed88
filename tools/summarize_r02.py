"""Summarise the round-2 ncu captures (tools/capture_r02.sh) into
profiles/r02/ncu_summary.json and refresh profiles/ncu_traffic.json (the DRAM
bytes per launch bench.py reports as roofline.traffic).
usage: python tools/summarize_r02.py gpurun_out/r02"""
import csv
import json
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEEP = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__grid_size", "launch__registers_per_thread", "smsp__inst_executed.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum"]
WHAT = {"cfg1_step": ("configs[1]", "configs[1] step kernel (DirectIPC, P=1, bench.py --mode p2p)"),
        "cfg1_window": ("configs[1]-window", "configs[1] through the window protocol (DDT_SELF_VIA_WINDOW=1)"),
        "comb": ("configs[3]", "configs[3] COMB 26-neighbour P=1 (paired x faces)"),
        "sparse32": ("configs[2]", "configs[2] sparse hindexed, B=32"),
        "dense4m": ("configs[4]", "configs[4] dense vector pack, 4 MiB x 64")}


def raw(path):
    rows = list(csv.reader(open(path)))
    return {h: (v, u) for h, v, u in zip(rows[0], rows[2], rows[1])}


def num(v):
    try:
        return float(v.replace(",", ""))
    except ValueError:
        return v


def main(d):
    out, traffic = {}, json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
    for name, (cfg, desc) in WHAT.items():
        p = os.path.join(d, f"{name}_raw.csv")
        if not os.path.exists(p):
            continue
        r = raw(p)
        m = {k: {"value": num(r[k][0]), "unit": r[k][1]} for k in KEEP if k in r}
        m["kernel"] = r.get("Kernel Name", ("?",))[0]
        m["what"] = desc
        dur_ns = m["gpu__time_duration.sum"]["value"] * (1e3 if m["gpu__time_duration.sum"]["unit"] == "us" else 1)
        byt = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            v, u = m[k]["value"], m[k]["unit"]
            byt += v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
        m["dram_bytes_per_launch"] = byt
        m["dram_GBps"] = round(byt / dur_ns, 1)
        out[name] = m
        traffic.setdefault(cfg, {})["ddt_fused_*" if "window" not in name else "ddt_exchange_*"] = byt
    # launch list of the bench command: mean duration per kernel name
    lp = os.path.join(d, "launches_bench.csv")
    if os.path.exists(lp):
        rows = list(csv.reader(open(lp)))
        hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
        hdr = rows[hi]
        ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
        agg = defaultdict(list)
        for r in rows[hi + 1:]:
            if len(r) > vi:
                agg[r[ki][:80]].append(num(r[vi]))
        out["launch_list_bench"] = {
            "command": "ncu --metrics gpu__time_duration.sum --clock-control none -c 400 python bench.py --steps 100 "
                       "--warmup 5 --no-extras --mode p2p",
            "note": "cold, serialised per-launch times (ncu replays each launch alone); only the share of the step "
                    "kernels is comparable with the bench's pipelined K-step graph",
            "kernels": {k: {"launches": len(v), "mean_ns": round(sum(v) / len(v), 1)} for k, v in agg.items()}}
    json.dump(out, open(os.path.join(ROOT, "profiles", "r02", "ncu_summary.json"), "w"), indent=1)
    json.dump(traffic, open(os.path.join(ROOT, "profiles", "ncu_traffic.json"), "w"), indent=1)
    print(json.dumps({k: (v.get("dram_GBps"), v.get("gpu__time_duration.sum")) for k, v in out.items()
                      if isinstance(v, dict) and "dram_GBps" in v}))


if __name__ == "__main__":
    main(sys.argv[1])
