"""Summarise the ncu captures of tools/capture_profiles.sh into profiles/<round>/
(ncu_summary.json, launch-list summaries) and profiles/ncu_traffic.json (per-launch
DRAM bytes read + written, read by bench.py for roofline.traffic)."""
import csv
import collections
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "prof_r")
rnd = sys.argv[2] if len(sys.argv) > 2 else "r01"
out_root = sys.argv[3] if len(sys.argv) > 3 else os.path.join(ROOT, "profiles")  # run on the box: gpurun_out/...
dst = os.path.join(out_root, rnd)
os.makedirs(dst, exist_ok=True)
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__grid_size", "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "sm__cycles_active.max", "gpc__cycles_elapsed.max"]
UNIT_SCALE = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1.0, "usecond": 1.0, "nsecond": 1e-3, "msecond": 1e3}
summary, traffic = {}, {}
for name, wl in [("full_cfg2", "configs[1]"), ("full_cfg3", "configs[2]"), ("full_cfg3cm", "configs[2]-cm"),
                 ("full_cfg4", "configs[3]"), ("full_cfg5", "configs[4]")]:
    rep = os.path.join(src, name + ".ncu-rep")
    if not os.path.exists(rep):
        continue
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    for row in rows[2:]:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        rec = {"kernel": d.get("Kernel Name")}
        for k in KEYS:
            v = d.get(k)
            try:
                v = float(str(v).replace(",", ""))
            except (TypeError, ValueError):
                pass
            rec[k] = v
            rec[k + ".unit"] = u.get(k)
        stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v.replace(",", "") or 0)
                  for k, v in d.items() if k.startswith("smsp__pcsamp_warps_issue_stalled_")
                  and not k.endswith("_not_issued") and v}
        tot = sum(stalls.values()) or 1.0
        rec["stall_share_top"] = {k: round(v / tot, 3) for k, v in sorted(stalls.items(), key=lambda kv: -kv[1])[:6]}
        rb = rec["dram__bytes_read.sum"] * UNIT_SCALE.get(rec["dram__bytes_read.sum.unit"], 1.0)
        wb = rec["dram__bytes_write.sum"] * UNIT_SCALE.get(rec["dram__bytes_write.sum.unit"], 1.0)
        rec["dram_bytes_per_launch"] = rb + wb
        summary[wl] = rec
        kfam = "ddt_exchange_*" if "exchange" in rec["kernel"] else "ddt_fused_*"
        traffic.setdefault(wl, {})[kfam] = rb + wb
launch = {}
for f in sorted(os.listdir(src)):
    if not f.startswith("launches_") or not f.endswith(".csv"):
        continue
    hdr, agg = None, collections.defaultdict(list)
    for r in csv.reader(open(os.path.join(src, f))):
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            agg[d["Kernel Name"][:60]].append(float(d["Metric Value"].replace(",", "")))
    launch[f] = {k: {"n": len(v), "mean_us": round(sum(v) / len(v) / 1e3, 3), "min_us": round(min(v) / 1e3, 3),
                     "share_of_listed_time": round(sum(v) / sum(sum(x) for x in agg.values()), 3)}
                 for k, v in agg.items()}
json.dump({"full_captures": summary, "launch_lists": launch}, open(os.path.join(dst, "ncu_summary.json"), "w"),
          indent=1)
json.dump(traffic, open(os.path.join(out_root, "ncu_traffic.json"), "w"), indent=1)
print(json.dumps({"full_captures": {k: {kk: v[kk] for kk in ("kernel", "gpu__time_duration.sum", "dram_bytes_per_launch")}
                                    for k, v in summary.items()}, "launch_lists": launch}, indent=1))
