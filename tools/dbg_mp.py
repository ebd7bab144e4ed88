"""Debug driver (scratch): 2 processes on one GPU, p2p exchange of a small
26-direction halo; prints per-iteration mismatch classification."""
import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from mp_util import free_port, init


def worker(rank, world, port, env, q):
    for k, v in env.items():
        os.environ[k] = v
    init(rank, world, port)
    import torch, torch.distributed as dist
    torch.cuda.set_device(0)
    import paper_conf_cluster_chukzsp20_b200 as ddt
    from ddt_inputs import halo_messages, proc_grid, global_block, padded_block, ghost_mask, random_bytes, ALL_DIRS
    P = world; grid = proc_grid(P); local = (6, 5, 7); G = tuple(n * g for n, g in zip(local, grid)); nvars = 2
    arrs = [torch.zeros(tuple(n + 2 for n in local), dtype=torch.int64, device="cuda") for _ in range(nvars)]
    msgs = halo_messages(rank, P, local, dirs=ALL_DIRS, nvars=nvars)
    sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
    comm = ddt.Comm.from_torch(0, nccl=False); qq = ddt.Queue()
    h = ddt.Halo(qq, comm, sends, recvs, mode="p2p", graph=False)
    gm = ghost_mask(local, ALL_DIRS)
    out = []
    prev = None
    for it in range(3):
        globs = [random_bytes(int(np.prod(G)) * 8, 900 + 10 * it + v).view(np.int64).reshape(G) for v in range(nvars)]
        for v, a in enumerate(arrs):
            a[1:-1, 1:-1, 1:-1] = torch.from_numpy(np.ascontiguousarray(global_block(globs[v], rank, P))).cuda()
        torch.cuda.synchronize(); dist.barrier()
        err = None
        try:
            h.exchange()
        except Exception as e:
            err = str(e)
        torch.cuda.synchronize(); dist.barrier()
        info = []
        exps = [padded_block(globs[v], rank, P) for v in range(nvars)]
        for v, a in enumerate(arrs):
            got = a.cpu().numpy(); exp = exps[v]
            bad = (got != exp) & gm
            n = int(bad.sum())
            cls = {}
            if n:
                gv = got[bad]
                cls["zero"] = int((gv == 0).sum())
                if prev is not None:
                    cls["prev_it"] = int((gv == prev[v][bad]).sum())
                    cls["prev_other_var"] = int((gv == prev[1 - v][bad]).sum())
                cls["other_var"] = int((gv == exps[1 - v][bad]).sum())
                cls["where"] = sorted(set(map(tuple, np.argwhere(bad)[:, :1].tolist())))[:4]
            info.append((n, cls))
        prev = exps
        out.append((it, err, info))
    q.put((rank, out))


if __name__ == "__main__":
    import torch.multiprocessing as mp
    envs = [{"DDT_GROUP_ALWAYS": "1"}, {"DDT_GROUP_ALWAYS": "1", "DDT_XSTATIC": "1"},
            {"DDT_GROUP_ALWAYS": "1", "DDT_XGRID_MODE": "2"}]
    for env in envs:
        ctx = mp.get_context("spawn"); q = ctx.Queue(); port = free_port()
        ps = [ctx.Process(target=worker, args=(r, 2, port, env, q)) for r in range(2)]
        [p.start() for p in ps]
        res = [q.get(timeout=300) for _ in range(2)]
        [p.join(60) for p in ps]
        for r in sorted(res):
            print(env, r, flush=True)
