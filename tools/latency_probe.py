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


if __name__ == "__main__":
    main()
