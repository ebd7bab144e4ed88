"""Diagnostic: halo exchange vs oracle on small grids, both modes; prints mismatch locations."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_cluster_chukzsp20_b200 as ddt
from ddt_inputs import halo_messages, FACE_DIRS, ALL_DIRS, random_bytes

def run(local, dirs, mode, graph):
    shape = tuple(n + 2 for n in local)
    a = torch.from_numpy(random_bytes(int(np.prod(shape)) * 8, 7).view(np.int64).reshape(shape).copy()).cuda()
    ref = a.cpu().numpy().copy()
    q = ddt.Queue(0)
    msgs = halo_messages(0, 1, local, dirs=dirs)
    sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), a, 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), a, 1) for m in msgs]
    comm = ddt.Comm.single(0)
    h = ddt.Halo(q, comm, sends, recvs, mode=mode, graph=graph)
    h.exchange(); torch.cuda.synchronize()
    by_tag = {m["recv_tag"]: m for m in msgs}
    omsgs = [dict(src_rank=0, dst_rank=0, var=0, send=oracle.Type(m["send_spec"]), recv=oracle.Type(by_tag[m["tag"]]["recv_spec"])) for m in msgs]
    arrays = {(0, 0): ref}
    oracle.exchange(arrays, omsgs)
    got = a.cpu().numpy()
    bad = np.argwhere(got != ref)
    print(local, len(dirs), mode, graph, "mismatches:", len(bad), bad[:10].tolist(), flush=True)
    h.destroy(); comm.close(); q.destroy()

for local in [(6, 7, 8), (9, 4, 3), (5, 6, 7)]:
    for dirs in [FACE_DIRS, ALL_DIRS]:
        for mode in ["nccl", "p2p"]:
            run(local, dirs, mode, False)
