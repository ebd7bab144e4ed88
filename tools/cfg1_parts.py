"""configs[1] step split by face kind (diagnostic): the bench harness (K-step
graph over 96 replicas, L2 read sweep) for all 6 faces, the 4 dense y/z faces
alone, the 2 x faces alone, and 1 face of each kind."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import FACE_DIRS  # noqa: E402

torch.cuda.set_device(0)
s = torch.cuda.Stream()
torch.cuda.set_stream(s)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
sets = {"all6": FACE_DIRS, "dense_yz4": [d for d in FACE_DIRS if d[2] == 0], "x2": [d for d in FACE_DIRS if d[2] != 0],
        "z2": [(1, 0, 0), (-1, 0, 0)], "y2": [(0, 1, 0), (0, -1, 0)]}
out = {}
for rep in range(2):
    for name, dirs in sets.items():
        wl = bench.HaloWorkload(ddt, torch, 0, 1, (128, 128, 128), dirs, 1, "p2p", ddt.Comm.single(0), 2, replicas=96,
                                graph=False)
        ms, _ = bench.run_steps(torch, wl, 500, 20, False, None, capture=True, flush_buf=flush)
        out.setdefault(name, []).append(round(ms * 1e3, 3))
        wl.close()
        torch.cuda.empty_cache()
print(json.dumps(out))
