"""N > 1 host logic on CPU: real multi-process runs over torch.distributed/gloo
(world size 2 and 4, 127.0.0.1).

* the host all-gather callback that carries halo-plan metadata into the C
  library (ddt_comm_t.host_allgather) returns every rank's bytes in rank order;
* the halo message recipe pairs correctly across real processes: every rank
  packs its sends with the CPU oracle, ships them with gloo isend/irecv keyed
  by (peer, tag), unpacks into its ghost layer, and the result equals
  np.pad(global, 1, mode="wrap") on every rank (Alg 3).
"""
import ctypes
import sys
import os

import numpy as np
import pytest

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from mp_util import free_port, init  # noqa: E402


def _allgather_worker(rank, world, port, q):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    init(rank, world, port)
    from paper_conf_cluster_chukzsp20_b200.halo import torch_allgather, _c_allgather
    cb = _c_allgather(torch_allgather())
    n = 24
    send = (ctypes.c_uint8 * n)(*[(rank * 31 + i) % 256 for i in range(n)])
    recv = (ctypes.c_uint8 * (n * world))()
    rc = cb(None, ctypes.addressof(send), n, ctypes.addressof(recv))
    ok = rc == 0 and all(recv[r * n + i] == (r * 31 + i) % 256 for r in range(world) for i in range(n))
    q.put((rank, ok))
    import torch.distributed as dist
    dist.destroy_process_group()


def _halo_worker(rank, world, port, faces_only, q):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    init(rank, world, port)
    import torch
    import torch.distributed as dist
    import oracle
    from ddt_inputs import (halo_messages, proc_grid, global_block, padded_block, ghost_mask, random_bytes,
                            FACE_DIRS, ALL_DIRS)
    P = world
    grid = proc_grid(P)
    local = (3, 4, 5)
    G = tuple(n * g for n, g in zip(local, grid))
    nvars = 2
    dirs = FACE_DIRS if faces_only else ALL_DIRS
    ok = True
    for v in range(nvars):
        glob = random_bytes(int(np.prod(G)) * 8, 500 + v).view(np.uint64).reshape(G)
        a = np.full(tuple(n + 2 for n in local), 0xA5A5A5A5A5A5A5A5, np.uint64)
        a[1:-1, 1:-1, 1:-1] = global_block(glob, rank, P)
        msgs = [m for m in halo_messages(rank, P, local, dirs=dirs, nvars=nvars) if m["var"] == v]
        reqs, bufs = [], []
        for m in msgs:  # post receives first (Alg 3 lines 5-6)
            o = oracle.Type(m["recv_spec"])
            buf = torch.empty(o.size, dtype=torch.uint8)
            bufs.append((m, o, buf))
            reqs.append(dist.irecv(buf, src=m["recv_peer"], tag=m["recv_tag"]) if m["recv_peer"] != rank else None)
        self_packed = {}
        for m in msgs:
            pk = oracle.pack(oracle.Type(m["send_spec"]), a)
            if m["peer"] == rank:
                self_packed[m["tag"]] = pk
            else:
                reqs.append(dist.isend(torch.from_numpy(pk), dst=m["peer"], tag=m["tag"]))
        for r in reqs:
            if r is not None:
                r.wait()
        for m, o, buf in bufs:
            data = self_packed[m["recv_tag"]] if m["recv_peer"] == rank else buf.numpy()
            oracle.unpack(o, data, a)
        exp = padded_block(glob, rank, P)
        gm = ghost_mask(local, dirs)
        ok &= bool(np.array_equal(a[gm], exp[gm]))
        ok &= bool(np.array_equal(a[1:-1, 1:-1, 1:-1], exp[1:-1, 1:-1, 1:-1]))
    q.put((rank, ok))
    dist.barrier()
    dist.destroy_process_group()


def _spawn(fn, world, *args):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=fn, args=(r, world, port) + args + (q,)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        r, ok = q.get(timeout=240)
        res[r] = ok
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return res


@pytest.mark.timeout(300)
def test_host_allgather_callback_world2():
    res = _spawn(_allgather_worker, 2)
    assert res == {0: True, 1: True}


@pytest.mark.timeout(300)
@pytest.mark.parametrize("world,faces_only", [(2, True), (2, False), (4, False)])
def test_halo_recipe_across_processes_gloo(world, faces_only):
    res = _spawn(_halo_worker, world, faces_only)
    assert all(res.values()) and len(res) == world
