"""General-list layouts (irregular block lengths -> GENERAL_LIST: per-vector
segment lookup) vs uniform lists of the same density: fused pack of B = 32
requests of a hindexed type with 1e5 blocks over 2^20 points, block lengths
uniform (3 floats) or irregular (1..5 floats, mean 3).  Persistent plan,
CUDA-event timed, L2 flushed before each launch.  Prints one JSON line per case."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402


def spec_for(irregular: bool, nblocks=100000, npoints=1 << 20, seed=7):
    rng = np.random.default_rng(seed)
    idx = np.sort(rng.choice(npoints - 8, nblocks, replace=False))
    if irregular:
        lens = rng.integers(1, 6, nblocks)
    else:
        lens = np.full(nblocks, 3)
    # hindexed of floats: block i = lens[i] floats at byte 12 * idx[i] (blocks may not overlap: clip)
    disp = 12 * idx
    gaps = np.diff(np.append(disp, 12 * npoints)) // 4
    lens = np.minimum(lens, gaps)
    return ("hindexed", [int(x) for x in lens], [int(x) for x in disp], ("basic", "float")), 12 * npoints + 64


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    for irregular in (False, True):
        spec, fp = spec_for(irregular)
        t = ddt.Type.from_spec(spec)
        B = 32
        src = torch.randint(0, 255, (B, fp), dtype=torch.uint8, device="cuda")
        dst = torch.empty((B, t.size), dtype=torch.uint8, device="cuda")
        q = ddt.Queue()
        for b in range(B):
            q.pack(t, src[b], 1, dst[b])
        plan = ddt.Plan(q)
        for _ in range(3):
            plan.launch()
        times = []
        for k in range(20):
            flush.fill_(k)
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            plan.launch()
            e.record(s)
            torch.cuda.synchronize()
            times.append(a.elapsed_time(e) * 1e3)
        us = statistics.median(times)
        print(json.dumps({"layout": t.layout_kind, "irregular": irregular, "segments": t.num_segments,
                          "packed_bytes": t.size, "batch": B, "us": round(us, 2),
                          "alg_gbs": round(2 * B * t.size / us / 1e3, 1)}), flush=True)
        plan.destroy()
        q.destroy()


if __name__ == "__main__":
    main()
