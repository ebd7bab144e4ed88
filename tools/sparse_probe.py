"""configs[2] sparse hindexed packs (B x 10^5 x 12-B blocks): kernel time of a
persistent plan after an L2 read sweep (clean L2, no dirty lines), for a set
of knob variants built side by side and timed round-robin (medians).
usage: python tools/sparse_probe.py [B]   (VARIANTS env: comma list of names)"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import config3_spec  # noqa: E402

VARIANTS = {
    "default": {},
    "rounds1": {"DDT_SEG_ROUNDS": "1"},
    "rounds4": {"DDT_SEG_ROUNDS": "4"},
    "noseg": {"DDT_NO_SEG": "1"},
    "grid0": {"DDT_GRID_MODE": "0"},
    "grid1": {"DDT_GRID_MODE": "1"},
}
KNOBS = ("DDT_SEG_ROUNDS", "DDT_NO_SEG", "DDT_GRID_MODE")


def main():
    B = int(sys.argv[1]) if len(sys.argv) > 1 else 32
    names = os.environ.get("VARIANTS", ",".join(VARIANTS)).split(",")
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    res = {}
    for order in ("sorted", "shuffled"):
        spec, nb = config3_spec(shuffled=(order == "shuffled"))
        t = ddt.Type.from_spec(spec)
        src = torch.empty((B, nb), dtype=torch.uint8, device="cuda")
        src.random_(0, 256)
        dst = torch.empty((B, t.size), dtype=torch.uint8, device="cuda")
        plans = {}
        base = dict(os.environ)
        for n in names:
            for k in KNOBS:
                os.environ.pop(k, None)
            os.environ.update(VARIANTS[n])
            ddt.reload_env()
            q = ddt.Queue()
            q.enqueue_many("pack", t, list(src), 1, list(dst))
            plans[n] = (q, ddt.Plan(q))
        os.environ.clear()
        os.environ.update(base)
        ddt.reload_env()
        times = {n: [] for n in names}
        s = torch.cuda.current_stream()
        for rep in range(15):
            for n in names:
                bench.l2_evict(torch, flush)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                plans[n][1].launch()
                b.record(s)
                torch.cuda.synchronize()
                times[n].append(a.elapsed_time(b) * 1e3)
        res[order] = {n: round(statistics.median(v[3:]), 2) for n, v in times.items()}
        for q, p in plans.values():
            p.destroy()
            q.destroy()
    print(json.dumps({"B": B, "us": res}))


if __name__ == "__main__":
    main()
