"""Launch a configs[4] dense-pack plan N times (for ncu captures).
usage: python tools/run_pack.py S B iters"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import config5_spec  # noqa: E402

S, B, iters = (int(x) for x in sys.argv[1:4])
torch.cuda.set_device(0)
spec, fp = config5_spec(S)
t = ddt.Type.from_spec(spec)
src = torch.empty((B, fp), dtype=torch.uint8, device="cuda")
src.random_(0, 256)
dst = torch.empty((B, S), dtype=torch.uint8, device="cuda")
q = ddt.Queue()
for b in range(B):
    q.pack(t, src[b], 1, dst[b])
plan = ddt.Plan(q)
for _ in range(iters):
    plan.launch()
torch.cuda.synchronize()
print("ok", S, B, iters)
