"""Summarise ncu raw CSV pages (one kernel each): duration, DRAM bytes and
throughput, L2 traffic, warp-stall breakdown.  usage: python tools/ncu_brief.py a_raw.csv [b_raw.csv ...]"""
import csv
import sys

KEYS = [("gpu__time_duration.sum", "dur"), ("dram__bytes_read.sum", "dram_rd"), ("dram__bytes_write.sum", "dram_wr"),
        ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram_%"),
        ("lts__t_bytes.sum", "l2_bytes"), ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%"),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "occ_%"),
        ("launch__grid_size", "grid"), ("launch__registers_per_thread", "regs"),
        ("smsp__inst_executed.sum", "inst")]


def load(path):
    rows = list(csv.reader(open(path)))
    hdr, units = rows[0], rows[1]
    vals = rows[2]
    return {h: (v, u) for h, v, u in zip(hdr, vals, units)}


for p in sys.argv[1:]:
    d = load(p)
    print(p.split("/")[-1], d.get("Kernel Name", ("?",))[0][:60])
    for k, n in KEYS:
        if k in d:
            print(f"  {n:9s} {d[k][0]:>16s} {d[k][1]}")
    st = {k: float(v[0].replace(",", "")) for k, v in d.items()
          if k.startswith("smsp__average_warp_latency_issue_stalled_") or
          (k.startswith("smsp__warp_issue_stalled_") and k.endswith("_per_warp_active.pct"))}
    tot = sum(st.values()) or 1
    top = sorted(st.items(), key=lambda kv: -kv[1])[:6]
    print("  stalls:", ", ".join(f"{k.replace('smsp__warp_issue_stalled_', '').replace('_per_warp_active.pct', '')}"
                                f"={v:.1f}" for k, v in top))
