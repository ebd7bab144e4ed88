"""Launch a fused pack plan N times (for ncu captures).
usage: python tools/run_pack.py S B iters          (configs[4] dense vector of S bytes, batch B)
       python tools/run_pack.py cfg3 B iters       (configs[2] sparse hindexed, batch B)
       python tools/run_pack.py cfg3cm B iters     (specfem3D_cm-style struct-on-indexed, batch B)
       ... [unpack]                                 (the unpack batch of the same layout instead)"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import config5_spec, config3_spec, config3_cm_spec  # noqa: E402

what, B, iters = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
unpack = len(sys.argv) > 4 and sys.argv[4] == "unpack"
torch.cuda.set_device(0)
if what == "cfg3":
    spec, fp = config3_spec()
elif what == "cfg3cm":
    spec, fp = config3_cm_spec()
else:
    spec, fp = config5_spec(int(what))
t = ddt.Type.from_spec(spec)
src = torch.empty((B, fp), dtype=torch.uint8, device="cuda")
src.random_(0, 256)
dst = torch.empty((B, t.size), dtype=torch.uint8, device="cuda")
q = ddt.Queue()
for b in range(B):
    if unpack:
        q.unpack(t, dst[b], 1, src[b])
    else:
        q.pack(t, src[b], 1, dst[b])
plan = ddt.Plan(q)
for _ in range(iters):
    plan.launch()
torch.cuda.synchronize()
print("ok", what, B, iters, "unpack" if unpack else "pack")
