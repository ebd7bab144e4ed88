"""Run N exchanges of a halo workload on one GPU (for ncu / nsight captures).
usage: python tools/run_halo.py {cfg2|cfg4} [mode] [iters]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import halo_messages, FACE_DIRS, ALL_DIRS  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
mode = sys.argv[2] if len(sys.argv) > 2 else "nccl"
iters = int(sys.argv[3]) if len(sys.argv) > 3 else 5
local, dirs, nvars = ((128,) * 3, FACE_DIRS, 1) if cfg == "cfg2" else ((512,) * 3, ALL_DIRS, 4)
torch.cuda.set_device(0)
arrs = [torch.zeros(tuple(n + 2 for n in local), dtype=torch.int64, device="cuda") for _ in range(nvars)]
msgs = halo_messages(0, 1, local, dirs=dirs, nvars=nvars)
cache = {}


def T(spec):
    k = repr(spec)
    if k not in cache:
        cache[k] = ddt.Type.from_spec(spec)
    return cache[k]


sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
q = ddt.Queue()
h = ddt.Halo(q, ddt.Comm.single(0), sends, recvs, mode=mode, graph=False)
for _ in range(iters):
    h.exchange()
torch.cuda.synchronize()
print("ok", cfg, mode, iters)
