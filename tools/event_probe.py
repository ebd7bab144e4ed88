"""K = 20 vs K = 500 with three ways of placing the timing events around the
K-step graph (configs[1], DirectIPC, 96 replicas, L2 read sweep first):
  A  stream events around g.replay() (bench.py run_steps);
  B  the two events captured INSIDE the graph (external event-record nodes);
  C  as B, with the L2 sweep captured in the graph too (no host gap at all).
Prints medians over rounds (diagnostic)."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
import bench  # noqa: E402
from ddt_inputs import FACE_DIRS  # noqa: E402


def main():
    torch.cuda.set_device(0)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    wl = bench.HaloWorkload(ddt, torch, 0, 1, (128, 128, 128), FACE_DIRS, 1, "p2p", ddt.Comm.single(0), 2,
                            replicas=96, graph=False)
    out = {}
    for K in (20, 500):
        for _ in range(5):
            wl.step()
        graphs = {}
        evs = {}
        for m in ("A", "B", "C"):
            g = torch.cuda.CUDAGraph()
            a = torch.cuda.Event(enable_timing=True, external=True)
            b = torch.cuda.Event(enable_timing=True, external=True)
            with torch.cuda.graph(g, stream=s):
                if m == "C":
                    flush.max()
                if m != "A":
                    a.record(s)
                for _ in range(K):
                    wl.step()
                if m != "A":
                    b.record(s)
            g.replay()
            torch.cuda.synchronize()
            graphs[m], evs[m] = g, (a, b)
        res = {m: [] for m in graphs}
        for _ in range(int(os.environ.get("ROUNDS", "9"))):
            for m, g in graphs.items():
                torch.cuda.synchronize()
                if m == "A":
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    flush.max()
                    a.record(s)
                    g.replay()
                    b.record(s)
                else:
                    a, b = evs[m]
                    if m == "B":
                        flush.max()
                    g.replay()
                torch.cuda.synchronize()
                res[m].append(a.elapsed_time(b) * 1e3 / K)
        out[K] = {m: {"median_us": round(statistics.median(v), 4), "min_us": round(min(v), 4)} for m, v in res.items()}
        print(K, json.dumps(out[K]), flush=True)
    for m in ("A", "B", "C"):
        print(m, "K20/K500", round(out[20][m]["median_us"] / out[500][m]["median_us"], 4))


if __name__ == "__main__":
    main()
