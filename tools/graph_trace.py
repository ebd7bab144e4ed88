"""CUPTI activity trace (torch.profiler / kineto; nsys is not in the image) of
bench.py's timed region for configs[1]: the K-step captured CUDA graph over R
rotating replicas, L2 read sweep first.  Every kernel of the replay with its
device start / end (ns), the gaps between consecutive step kernels, and the
per-step number that follows from them -- next to the CUDA-event value of an
identical un-profiled replay in the same process.

usage: python tools/graph_trace.py [K] [window]  -> JSON on stdout
  window: every self message through the multi-GPU window protocol
          (DDT_SELF_VIA_WINDOW=1) instead of DirectIPC."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if len(sys.argv) > 2 and sys.argv[2] == "window":
    os.environ["DDT_SELF_VIA_WINDOW"] = "1"
import torch  # noqa: E402
from torch.profiler import profile, ProfilerActivity  # noqa: E402

import bench  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import FACE_DIRS  # noqa: E402


def kernels(prof):
    out = []
    try:
        for e in prof.profiler.kineto_results.events():
            if e.device_type().name == "CUDA" and not e.name().startswith(("Memcpy", "Memset")):
                out.append((e.name(), int(e.start_ns()), int(e.start_ns() + e.duration_ns())))
    except Exception:
        for e in prof.events():
            if e.device_type.name == "CUDA":
                out.append((e.name, int(e.time_range.start * 1e3), int(e.time_range.end * 1e3)))
    return sorted(out, key=lambda x: x[1])


def main():
    K = int(sys.argv[1]) if len(sys.argv) > 1 else 20
    torch.cuda.set_device(0)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    wl = bench.HaloWorkload(ddt, torch, 0, 1, (128, 128, 128), FACE_DIRS, 1, "p2p", ddt.Comm.single(0), 2,
                            replicas=96, graph=False)
    for _ in range(5):
        wl.step()
    first = wl.k  # the first captured (timed) step's replica
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(K):
            wl.step()
    g.replay()
    torch.cuda.synchronize()
    ev_ms = []
    for _ in range(5):  # CUDA-event view, exactly bench.run_steps' timed region
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        bench.l2_evict(torch, flush)
        wl.step_at(first - 1)  # bench.run_steps: the code-warming step on a non-timed replica
        a.record(s)
        g.replay()
        b.record(s)
        torch.cuda.synchronize()
        ev_ms.append(a.elapsed_time(b) / K)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        bench.l2_evict(torch, flush)
        wl.step_at(first - 1)
        g.replay()
        torch.cuda.synchronize()
    ks = kernels(prof)
    steps = [k for k in ks if "ddt_" in k[0]]
    if len(steps) == K + 1:
        steps = steps[1:]  # the untimed code-warming step before the replay
    other = [k for k in ks if "ddt_" not in k[0]]
    dur = [(e - st) / 1e3 for _, st, e in steps]
    gaps = [(steps[i + 1][1] - steps[i][2]) / 1e3 for i in range(len(steps) - 1)]
    starts = [(steps[i + 1][1] - steps[i][1]) / 1e3 for i in range(len(steps) - 1)]
    span = (steps[-1][2] - steps[0][1]) / 1e3 if steps else 0.0
    res = {"workload": "configs[1] 128^3 faces, P=1, " + ("window protocol" if os.environ.get("DDT_SELF_VIA_WINDOW")
                                                          else "DirectIPC"),
           "K": K, "replicas": 96, "kernels_in_replay": len(steps), "other_kernels": sorted({k[0] for k in other}),
           "kernel_name": steps[0][0] if steps else None,
           "per_step_us_from_trace": round(span / max(1, len(steps)), 3),
           "first_start_to_last_end_us": round(span, 3),
           "kernel_duration_us": {"median": round(statistics.median(dur), 3), "min": round(min(dur), 3),
                                  "max": round(max(dur), 3), "first": round(dur[0], 3)},
           "start_to_start_us": {"median": round(statistics.median(starts), 3)} if starts else None,
           "gap_end_to_next_start_us": {"median": round(statistics.median(gaps), 3),
                                        "min": round(min(gaps), 3)} if gaps else None,
           "note": ("kernels overlap their predecessor's tail under programmatic dependent launch, so a gap can be "
                    "negative; per-step = (last end - first start) / K"),
           "cuda_event_us_per_step": {"median": round(statistics.median(ev_ms) * 1e3, 3),
                                      "runs": [round(x * 1e3, 3) for x in ev_ms]},
           "kernels": [{"name": n[:60], "start_ns": st - steps[0][1], "end_ns": e - steps[0][1]}
                       for n, st, e in steps]}
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
