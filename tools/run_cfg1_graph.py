"""Replay bench.py's configs[1] K-step graph N times (for ncu --graph-profiling
graph: DRAM bytes of the pipelined steady state = graph total / K).
usage: python tools/run_cfg1_graph.py [K] [replays]"""
import os
import sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import FACE_DIRS  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 100
N = int(sys.argv[2]) if len(sys.argv) > 2 else 4
torch.cuda.set_device(0)
s = torch.cuda.Stream()
torch.cuda.set_stream(s)
wl = bench.HaloWorkload(ddt, torch, 0, 1, (128, 128, 128), FACE_DIRS, 1, "p2p", ddt.Comm.single(0), 2, replicas=96,
                        graph=False)
for _ in range(5):
    wl.step()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=s):
    for _ in range(K):
        wl.step()
for _ in range(N):
    g.replay()
torch.cuda.synchronize()
print("ok", K, N)
