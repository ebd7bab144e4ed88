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


def _worker_bytes(rank, world, port, opts, q):
    """Like _worker, but every rank's arrays live in uint8 device buffers at a
    byte offset (odd ranks at 4 mod 8 when opts['mis']: sender and receiver
    vector widths then differ, so messages are released whole -- the fan-out
    path), with optional env knobs, element type and local size."""
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    for k, v in opts.get("env", {}).items():
        os.environ[k] = v
    ok = False
    try:
        init(rank, world, port)
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(0)
        import paper_conf_cluster_chukzsp20_b200 as ddt
        from ddt_inputs import (halo_messages, proc_grid, global_block, padded_block, ghost_mask, random_bytes,
                                FACE_DIRS, ALL_DIRS)
        dirs = FACE_DIRS if opts["dirs"] == "faces" else ALL_DIRS
        P, local, nvars, base = world, tuple(opts["local"]), opts.get("nvars", 2), opts.get("base", "double")
        esz, dt = (8, np.int64) if base == "double" else (4, np.int32)
        grid = proc_grid(P)
        G = tuple(n * g for n, g in zip(local, grid))
        shape = tuple(n + 2 for n in local)
        nbytes = int(np.prod(shape)) * esz
        off = 4 if (opts.get("mis") and rank % 2 == 1) else 0
        bufs = [torch.full((nbytes + 64,), 0xA5, dtype=torch.uint8, device="cuda") for _ in range(nvars)]
        msgs = halo_messages(rank, P, local, dirs=dirs, nvars=nvars, base=base)
        cache = {}

        def T(spec):
            if repr(spec) not in cache:
                cache[repr(spec)] = ddt.Type.from_spec(spec)
            return cache[repr(spec)]
        sends = [(m["peer"], m["tag"], T(m["send_spec"]), (bufs[m["var"]], off), 1) for m in msgs]
        recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), (bufs[m["var"]], off), 1) for m in msgs]
        comm = ddt.Comm.from_torch(0, nccl=False)
        qq = ddt.Queue()
        graph = opts.get("graph", False)
        h = ddt.Halo(qq, comm, sends, recvs, mode=opts.get("mode", "p2p"), graph=graph)
        gm = ghost_mask(local, dirs)
        ok = True
        for it in range(opts.get("iters", 3)):
            globs = [random_bytes(int(np.prod(G)) * esz, 700 + 10 * it + v).view(dt).reshape(G) for v in range(nvars)]
            for v in range(nvars):
                a = np.full(shape, -1, dt)  # ghosts != any expected value pattern
                a[1:-1, 1:-1, 1:-1] = global_block(globs[v], rank, P)
                bufs[v][off:off + nbytes].copy_(torch.from_numpy(a.view(np.uint8).reshape(-1)))
            torch.cuda.synchronize()
            dist.barrier()
            h.exchange()
            torch.cuda.synchronize()
            dist.barrier()
            for v in range(nvars):
                got = bufs[v][off:off + nbytes].cpu().numpy().view(dt).reshape(shape)
                exp = padded_block(globs[v], rank, P)
                ok &= bool(np.array_equal(got[gm], exp[gm]))
                ok &= bool(np.array_equal(got[1:-1, 1:-1, 1:-1], exp[1:-1, 1:-1, 1:-1]))
        h.destroy()
        dist.barrier()
        comm.close()
        qq.destroy()
        dist.destroy_process_group()
    except Exception as e:
        print(f"rank {rank}: {type(e).__name__}: {e}", flush=True)
        ok = False
    q.put((rank, ok))


def _spawn(target, world, extra, timeout=400):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=target, args=(r, world, port) + extra + (q,)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(world):
            r, ok = q.get(timeout=timeout)
            res[r] = ok
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    return res


@pytest.mark.timeout(900)
@pytest.mark.parametrize("world,opts", [
    # the per-chunk flag protocol for every message (no LL)
    (2, dict(dirs="all", local=(6, 5, 7), env={"DDT_NO_LL": "1"}, iters=4)),
    (4, dict(dirs="all", local=(6, 5, 7), env={"DDT_NO_LL": "1"}, iters=3)),
    (8, dict(dirs="faces", local=(6, 5, 7), env={"DDT_NO_LL": "1"}, iters=2)),
    # messages > 512 KB (528 KiB z faces): per-chunk flags at 2 vectors per thread per item
    (2, dict(dirs="faces", local=(4, 260, 260), nvars=1, iters=3)),
    (2, dict(dirs="faces", local=(4, 260, 260), nvars=1, iters=4, graph=True)),
    # 4-B elements (4-B vectors, LL does not apply)
    (2, dict(dirs="all", local=(6, 10, 12), base="float", iters=3)),
    (4, dict(dirs="all", local=(6, 10, 12), base="float", iters=3)),
    # sender / receiver widths differ (odd ranks at 4 mod 8): whole-message fan-out + counters
    (2, dict(dirs="all", local=(6, 10, 12), mis=True, iters=3)),
    (4, dict(dirs="all", local=(12, 20, 24), mis=True, iters=3)),
    (2, dict(dirs="faces", local=(4, 260, 260), nvars=1, mis=True, iters=3)),
    # configs[1] at full size with P = 2 (remote z faces + self faces), both window formats
    (2, dict(dirs="faces", local=(128, 128, 128), nvars=1, iters=2)),
    (2, dict(dirs="faces", local=(128, 128, 128), nvars=1, iters=2, env={"DDT_NO_LL": "1"})),
    (2, dict(dirs="faces", local=(128, 128, 128), nvars=1, iters=2, mode="p2p_direct")),
    # one CTA per item forced for the exchange kernel (ticket-claimed)
    (2, dict(dirs="all", local=(12, 20, 24), iters=3, env={"DDT_XGRID_MODE": "2"})),
    # exchange pairs (+x / -x packs and unpacks in one item) between real processes
    (2, dict(dirs="all", local=(12, 20, 24), iters=3, env={"DDT_XPAIR_ALWAYS": "1"})),
    (8, dict(dirs="all", local=(6, 10, 12), iters=2, env={"DDT_XPAIR_ALWAYS": "1", "DDT_NO_LL": "1"})),
    # resident grid claiming chunks (the multi-wave launch form) with per-chunk flags, whole-message
    # counters and the pack-free protocol: every message keeps its own item size (xub_for)
    (2, dict(dirs="all", local=(24, 40, 48), iters=3, mode="p2p_direct", env={"DDT_XGRID_MODE": "1"})),
    (2, dict(dirs="all", local=(24, 40, 48), iters=3, mode="p2p_direct", mis=True, env={"DDT_XGRID_MODE": "1"})),
    (2, dict(dirs="all", local=(24, 40, 48), iters=3, mis=True, env={"DDT_XGRID_MODE": "1", "DDT_NO_LL": "1"})),
])
def test_exchange_protocols_multiprocess(world, opts):
    res = _spawn(_worker_bytes, world, (opts,))
    assert len(res) == world and all(res.values()), res


def _bad_args_worker(rank, world, port, q):
    """Rank 1 passes an invalid message (peer out of range); rank 0 is valid.
    Both must fail ddt_halo_create (the local checks are agreed before any
    collective metadata round), neither may hang."""
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    res = "none"
    try:
        init(rank, world, port)
        import torch
        torch.cuda.set_device(0)
        import paper_conf_cluster_chukzsp20_b200 as ddt
        from ddt_inputs import halo_messages, FACE_DIRS
        local = (4, 5, 6)
        a = torch.zeros(tuple(n + 2 for n in local), dtype=torch.int64, device="cuda")
        msgs = halo_messages(rank, world, local, dirs=FACE_DIRS)
        sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), a, 1) for m in msgs]
        recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), a, 1) for m in msgs]
        if rank == 1:
            p, t, ty, b, c = sends[0]
            sends[0] = (world + 3, t, ty, b, c)
        comm = ddt.Comm.from_torch(0, nccl=False)
        qq = ddt.Queue()
        try:
            ddt.Halo(qq, comm, sends, recvs, mode="p2p", graph=False)
            res = "created"
        except Exception as e:
            res = f"error:{e}"
    except Exception as e:
        res = f"setup:{type(e).__name__}: {e}"
    q.put((rank, res))


@pytest.mark.timeout(300)
def test_halo_create_fails_on_every_rank_together():
    res = _spawn(_bad_args_worker, 2, (), timeout=200)
    assert len(res) == 2, res
    assert all(v.startswith("error:") for v in res.values()), res


def _occupied_worker(rank, world, port, q):
    """2 processes on one GPU: each holds all but one SM of its context with an
    occupier kernel (max shared carveout) on a side stream, then runs the P2P
    window exchange (per-chunk flags, DDT_NO_LL) with its peer; both must finish
    while their occupiers still run (processes time-slice the GPU)."""
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["DDT_NO_LL"] = "1"
    ok = False
    try:
        init(rank, world, port)
        import ctypes
        import time
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(0)
        import paper_conf_cluster_chukzsp20_b200 as ddt
        from gpu_util import occupier
        from ddt_inputs import halo_messages, proc_grid, global_block, padded_block, ghost_mask, random_bytes, ALL_DIRS
        P, local = world, (16, 40, 48)
        G = tuple(n * g for n, g in zip(local, proc_grid(P)))
        a = torch.zeros(tuple(n + 2 for n in local), dtype=torch.int64, device="cuda")
        msgs = halo_messages(rank, P, local, dirs=ALL_DIRS)
        sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), a, 1) for m in msgs]
        recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), a, 1) for m in msgs]
        comm = ddt.Comm.from_torch(0, nccl=False)
        qq = ddt.Queue()
        h = ddt.Halo(qq, comm, sends, recvs, mode="p2p", graph=False)
        h.set_timeout(20.0)
        gm = ghost_mask(local, ALL_DIRS)

        def fill(it):
            glob = random_bytes(int(np.prod(G)) * 8, 300 + it).view(np.int64).reshape(G)
            a[1:-1, 1:-1, 1:-1] = torch.from_numpy(np.ascontiguousarray(global_block(glob, rank, P))).cuda()
            torch.cuda.synchronize()
            return glob

        glob = fill(0)  # warm-up exchange: kernels loaded before the SMs are held
        dist.barrier()
        h.exchange()
        torch.cuda.synchronize()
        dist.barrier()
        ok = bool(np.array_equal(a.cpu().numpy()[gm], padded_block(glob, rank, P)[gm]))
        glob = fill(1)
        occ = occupier()
        nsm = torch.cuda.get_device_properties(0).multi_processor_count
        ctas = 2 * nsm - 1
        stop = torch.zeros(1, dtype=torch.int32).pin_memory()
        started = torch.zeros(ctas, dtype=torch.int32).pin_memory()
        s_occ = torch.cuda.Stream()
        assert occ.occupy_launch(ctypes.c_void_p(s_occ.cuda_stream), ctas, 1024, ctypes.c_void_p(stop.data_ptr()),
                                 ctypes.c_void_p(started.data_ptr()), int(60e9)) == 0
        t0 = time.time()
        while int(started.sum()) < ctas and time.time() - t0 < 20:
            time.sleep(0.001)
        ok &= int(started.sum()) == ctas
        dist.barrier()
        h.exchange()
        cur = torch.cuda.current_stream()
        t0 = time.time()
        while not cur.query() and time.time() - t0 < 40:
            time.sleep(0.002)
        finished = cur.query()
        still = not s_occ.query()
        stop[0] = 1
        torch.cuda.synchronize()
        ok &= finished and still
        dist.barrier()
        ok &= bool(np.array_equal(a.cpu().numpy()[gm], padded_block(glob, rank, P)[gm]))
        h.destroy()
        dist.barrier()
        comm.close()
        qq.destroy()
        dist.destroy_process_group()
    except Exception as e:
        print(f"rank {rank}: {type(e).__name__}: {e}", flush=True)
        ok = False
    q.put((rank, ok))


@pytest.mark.timeout(600)
def test_exchange_multiprocess_while_sms_are_held():
    res = _spawn(_occupied_worker, 2, (), timeout=300)
    assert len(res) == 2 and all(res.values()), res
