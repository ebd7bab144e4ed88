"""Latency floor probe (diagnostic, not a bench line): CUDA-event-timed cost of
(a) a graph replay of one trivial torch kernel, (b) a direct trivial launch,
(c) the configs[1] exchange (graph and direct), each with and without
per-iteration events."""
import os
import sys
import statistics

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import halo_messages, FACE_DIRS  # noqa: E402


def per_iter(fn, K=300, flush=None):
    s = torch.cuda.current_stream()
    for _ in range(20):
        fn()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for k in range(K):
        if flush is not None:
            flush.fill_(k & 255)
        ev[k][0].record(s)
        fn()
        ev[k][1].record(s)
    torch.cuda.synchronize()
    t = [a.elapsed_time(b) * 1e3 for a, b in ev]
    return statistics.median(t), sum(t) / len(t)


def back_to_back(fn, K=1000):
    s = torch.cuda.current_stream()
    for _ in range(20):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(K):
        fn()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3 / K


def main():
    torch.cuda.set_device(0)
    x = torch.zeros(1, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        x.add_(1)
    print("trivial graph replay   per-iter (p50, mean) us:", per_iter(g.replay), " b2b:", back_to_back(g.replay))
    print("trivial direct launch  per-iter (p50, mean) us:", per_iter(lambda: x.add_(1)), " b2b:",
          back_to_back(lambda: x.add_(1)))
    local = (128, 128, 128)
    a = torch.zeros((130, 130, 130), dtype=torch.int64, device="cuda")
    msgs = halo_messages(0, 1, local, dirs=FACE_DIRS)
    sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), a, 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), a, 1) for m in msgs]
    for mode in ("nccl", "p2p"):
        for graph in (True, False):
            q = ddt.Queue()
            h = ddt.Halo(q, ddt.Comm.single(0), sends, recvs, mode=mode, graph=graph)
            print(f"exchange {mode:4s} graph={graph!s:5s} per-iter hot {per_iter(h.exchange)} cold "
                  f"{per_iter(h.exchange, flush=flush)} b2b {back_to_back(h.exchange):.2f}")
            h.destroy()
            q.destroy()
    rotating(sends, recvs, local)


def rotating(sends0, recvs0, local, R=64, K=640):
    """configs[1] exchanges over R independent 130^3 arrays (touched DRAM
    footprint R x ~3 MB > L2), K back to back: (a) host-issued launches,
    (b) captured K-exchange CUDA graph; plus a K-node graph of trivial kernels
    as the launch floor.  Per-exchange device time = total / K."""
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    msgs = halo_messages(0, 1, local, dirs=FACE_DIRS)
    q = ddt.Queue(stream=s)
    arrs, halos = [], []
    for r in range(R):
        a = torch.zeros((130, 130, 130), dtype=torch.int64, device="cuda")
        sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), a, 1) for m in msgs]
        recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), a, 1) for m in msgs]
        arrs.append(a)
        halos.append(ddt.Halo(q, ddt.Comm.single(0), sends, recvs, mode="p2p", graph=False))

    def host_loop():
        for k in range(K):
            halos[k % R].exchange()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    host_loop()
    torch.cuda.synchronize()
    ev[0].record(s)
    host_loop()
    ev[1].record(s)
    torch.cuda.synchronize()
    print(f"rotating R={R} host-issued b2b: {ev[0].elapsed_time(ev[1]) * 1e3 / K:.2f} us/exchange")
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for k in range(K):
            halos[k % R].exchange()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        ev[0].record(s)
        g.replay()
        ev[1].record(s)
        torch.cuda.synchronize()
        ts.append(ev[0].elapsed_time(ev[1]) * 1e3 / K)
    print(f"rotating R={R} K-exchange graph: {statistics.median(ts):.2f} us/exchange")
    x = torch.zeros(1, device="cuda")
    g2 = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g2, stream=s):
        for k in range(K):
            x.add_(1)
    g2.replay()
    torch.cuda.synchronize()
    ev[0].record(s)
    g2.replay()
    ev[1].record(s)
    torch.cuda.synchronize()
    print(f"trivial K-node graph: {ev[0].elapsed_time(ev[1]) * 1e3 / K:.2f} us/node")


if __name__ == "__main__":
    main()
