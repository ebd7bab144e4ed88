"""N > 1 on one GPU: P real processes (one rank each) share cuda:0 and run the
fused single-kernel P2P halo exchange through CUDA-IPC windows -- the multi-GPU
data path (pack stores into the peer's window, release flags, acquire-wait
unpack, double-buffered parity), with plan metadata carried by the host
all-gather over gloo.  Processes on one GPU are time-sliced, so this checks
correctness (several iterations, every rank vs np.pad wrap), not speed.
"""
import os
import sys

import numpy as np
import pytest

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from mp_util import free_port, init  # noqa: E402

pytestmark = pytest.mark.gpu


def _worker(rank, world, port, dirs_name, iters, mode, q, group=False):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    if group:  # interleave equal-size requests even in one-wave plans (halo.cpp make_table)
        os.environ["DDT_GROUP_ALWAYS"] = "1"
    ok = False
    try:
        init(rank, world, port)
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(0)
        import paper_conf_cluster_chukzsp20_b200 as ddt
        from ddt_inputs import (halo_messages, proc_grid, global_block, padded_block, ghost_mask, random_bytes,
                                FACE_DIRS, ALL_DIRS)
        dirs = FACE_DIRS if dirs_name == "faces" else ALL_DIRS
        P = world
        grid = proc_grid(P)
        local = (6, 5, 7)
        G = tuple(n * g for n, g in zip(local, grid))
        nvars = 2
        arrs = [torch.zeros(tuple(n + 2 for n in local), dtype=torch.int64, device="cuda") for _ in range(nvars)]
        for a in arrs:
            a.view(torch.uint8).fill_(0xA5)
        msgs = halo_messages(rank, P, local, dirs=dirs, nvars=nvars)
        cache = {}

        def T(spec):
            k = repr(spec)
            if k not in cache:
                cache[k] = ddt.Type.from_spec(spec)
            return cache[k]

        sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
        recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
        comm = ddt.Comm.from_torch(0, nccl=False)
        qq = ddt.Queue()
        h = ddt.Halo(qq, comm, sends, recvs, mode=mode, graph=(iters % 2 == 0))
        ok = True
        gm = ghost_mask(local, dirs)
        for it in range(iters):
            globs = [random_bytes(int(np.prod(G)) * 8, 900 + 10 * it + v).view(np.int64).reshape(G)
                     for v in range(nvars)]
            for v, a in enumerate(arrs):
                a[1:-1, 1:-1, 1:-1] = torch.from_numpy(np.ascontiguousarray(global_block(globs[v], rank, P))).cuda()
            torch.cuda.synchronize()
            dist.barrier()  # every rank's interior is written before anyone packs
            h.exchange()
            torch.cuda.synchronize()
            dist.barrier()  # nobody rewrites its interior while a peer may still read it
            for v, a in enumerate(arrs):
                got = a.cpu().numpy()
                exp = padded_block(globs[v], rank, P)
                ok &= bool(np.array_equal(got[gm], exp[gm]))
                ok &= bool(np.array_equal(got[1:-1, 1:-1, 1:-1], exp[1:-1, 1:-1, 1:-1]))
        h.destroy()
        dist.barrier()
        comm.close()
        qq.destroy()
        dist.destroy_process_group()
    except Exception as e:  # report instead of hanging the parent
        print(f"rank {rank}: {type(e).__name__}: {e}", flush=True)
        ok = False
    q.put((rank, ok))


@pytest.mark.timeout(600)
@pytest.mark.parametrize("world,dirs_name,iters,mode,group", [
    (2, "faces", 3, "p2p", False), (2, "all", 4, "p2p", False), (4, "all", 3, "p2p", False),
    (8, "faces", 2, "p2p", False), (2, "all", 4, "p2p_direct", False), (4, "all", 3, "p2p_direct", False),
    (8, "faces", 2, "p2p_direct", False), (2, "all", 4, "p2p", True), (4, "all", 3, "p2p", True),
    (4, "all", 3, "p2p_direct", True)])
def test_p2p_exchange_multiprocess_one_gpu(world, dirs_name, iters, mode, group):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, dirs_name, iters, mode, q, group))
             for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(world):
            r, ok = q.get(timeout=400)
            res[r] = ok
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    assert len(res) == world and all(res.values()), res
