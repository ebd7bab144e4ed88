"""Trace one fused P2P exchange (configs[1], or COMB with argument "comb"; self
messages through the window path, or with XMODE=direct through the pack-free
P2P_DIRECT protocol) and print the per-phase critical path (diagnostic)."""
import os
import sys
DIRECT = os.environ.get("XMODE") == "direct"
os.environ.setdefault("DDT_SELF_VIA_DIRECT" if DIRECT else "DDT_SELF_VIA_WINDOW", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import halo_messages, FACE_DIRS, ALL_DIRS  # noqa: E402

torch.cuda.set_device(0)
comb = len(sys.argv) > 1 and sys.argv[1] == "comb"
local = (512, 512, 512) if comb else (128, 128, 128)
nvars = 4 if comb else 1
arrs = [torch.zeros(tuple(n + 2 for n in local), dtype=torch.int64, device="cuda") for _ in range(nvars)]
msgs = halo_messages(0, 1, local, dirs=ALL_DIRS if comb else FACE_DIRS, nvars=nvars)
sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
h = ddt.Halo(ddt.Queue(), ddt.Comm.single(0), sends, recvs, mode="p2p_direct" if DIRECT else "p2p", graph=False)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(5):
    h.exchange()
torch.cuda.synchronize()
for it in range(3):
    read = h.trace(200000)
    flush.max()
    torch.cuda.synchronize()
    h.exchange()
    r = read()
    t = r["t0"].min()
    ph = {k: (r[k] - t) / 1e3 for k in ("t0", "t1", "t2", "t3")}
    print(f"iter {it}: records {len(r)}  span {ph['t3'].max():.2f} us  CTAs {len(set(r['cta'].tolist()))}")
    for name, m in (("pack", r["op"] == 0), ("unpack", r["op"] == 1), ("direct", r["op"] == 2),
                    ("signal", r["op"] == 3)):
        if m.any():
            print(f"  {name:6s} start [{ph['t0'][m].min():.2f}, {ph['t0'][m].max():.2f}]  wait-done max {ph['t1'][m].max():.2f}"
                  f"  data-done [{ph['t2'][m].min():.2f}, {ph['t2'][m].max():.2f}]  signal-done max {ph['t3'][m].max():.2f}"
                  f"  | per-item wait {np.median((r['t1']-r['t0'])[m])/1e3:.2f}  data {np.median((r['t2']-r['t1'])[m])/1e3:.2f}"
                  f"  signal {np.median((r['t3']-r['t2'])[m])/1e3:.2f} us (medians)")
