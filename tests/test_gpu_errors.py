"""Error paths through the C ABI on a GPU: mismatched halo plans are rejected at
create time, overlapping receive layouts are refused (R5), a type freed while a
request is in flight stays alive until the batch completes, and a P2P peer that
never enters the exchange produces DDT_ERR_TIMEOUT instead of a hang."""
import gc
import os
import sys

import numpy as np
import pytest

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from mp_util import free_port, init  # noqa: E402

import oracle  # noqa: E402
from ddt_inputs import random_bytes, config1_spec  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ddt():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_cluster_chukzsp20_b200.build import build
    build()
    import paper_conf_cluster_chukzsp20_b200 as m
    return m


def _halo(ddt, sends, recvs, mode):
    return ddt.Halo(ddt.Queue(), ddt.Comm.single(0), sends, recvs, mode=mode, graph=False)


@pytest.mark.parametrize("mode", ["nccl", "p2p"])
def test_halo_create_rejects_mismatches(ddt, mode):
    import torch
    a = torch.zeros(4096, dtype=torch.uint8, device="cuda")
    t8 = ddt.Type.from_spec(("vector", 8, 1, 2, ("basic", "double")))
    t4 = ddt.Type.from_spec(("vector", 4, 1, 2, ("basic", "double")))
    with pytest.raises(ddt.DDTError) as e:  # send tag 1 has no receive
        _halo(ddt, [(0, 1, t8, a, 1)], [(0, 2, t8, (a, 2048), 1)], mode)
    assert e.value.code == -8
    with pytest.raises(ddt.DDTError) as e:  # same tag, different packed sizes
        _halo(ddt, [(0, 1, t8, a, 1)], [(0, 1, t4, (a, 2048), 1)], mode)
    assert e.value.code == -8
    ov = ddt.Type.from_spec(("vector", 3, 2, 1, ("basic", "double")))  # blocks overlap
    sz = ddt.Type.from_spec(("contiguous", 6, ("basic", "double")))
    with pytest.raises(ddt.DDTError) as e:
        _halo(ddt, [(0, 1, sz, a, 1)], [(0, 1, ov, (a, 2048), 1)], mode)
    assert e.value.code == -4
    with pytest.raises(ddt.DDTError) as e:  # duplicate (peer, tag)
        _halo(ddt, [(0, 1, t8, a, 1), (0, 1, t8, (a, 512), 1)], [(0, 1, t8, (a, 2048), 1)], mode)
    assert e.value.code == -1


def test_type_freed_while_in_flight(ddt):
    import torch
    q = ddt.Queue()
    src_h = random_bytes(8192, 3)
    src = torch.from_numpy(src_h).cuda()
    dst = torch.zeros(512, dtype=torch.uint8, device="cuda")

    def enqueue_with_temporary_type():
        t = ddt.Type.from_spec(config1_spec())
        q.pack(t, src, 1, dst)
        # t goes out of scope: ddt_free drops the caller's reference (deferred, P:241 semantics)

    enqueue_with_temporary_type()
    gc.collect()
    q.wait()
    assert np.array_equal(dst.cpu().numpy(), oracle.pack(oracle.Type(config1_spec()), src_h))
    with pytest.raises(ddt.DDTError):
        q.query(10 ** 9)  # unknown uid
    q.destroy()


def _timeout_worker(rank, world, port, q):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    ok = False
    try:
        init(rank, world, port)
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(0)
        import paper_conf_cluster_chukzsp20_b200 as ddt
        from ddt_inputs import halo_messages, FACE_DIRS
        local = (4, 4, 4)
        a = torch.zeros((6, 6, 6), dtype=torch.int64, device="cuda")
        msgs = halo_messages(rank, world, local, dirs=FACE_DIRS)
        sends = [(m["peer"], m["tag"], ddt.Type.from_spec(m["send_spec"]), a, 1) for m in msgs]
        recvs = [(m["recv_peer"], m["recv_tag"], ddt.Type.from_spec(m["recv_spec"]), a, 1) for m in msgs]
        comm = ddt.Comm.from_torch(0, nccl=False)
        h = ddt.Halo(ddt.Queue(), comm, sends, recvs, mode="p2p", graph=False)
        if rank == 0:
            h.set_timeout(0.2)
            h.exchange()  # rank 1 never enters: every wait expires after 0.2 s
            torch.cuda.synchronize()
            try:
                h.exchange()
            except ddt.DDTError as e:
                ok = e.code == -9
        else:
            ok = True
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:
        print(f"rank {rank}: {type(e).__name__}: {e}", flush=True)
    q.put((rank, ok))


@pytest.mark.timeout(300)
def test_p2p_wait_times_out_instead_of_hanging():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_timeout_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(2):
            r, ok = q.get(timeout=200)
            res[r] = ok
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    assert res == {0: True, 1: True}, res


def test_flush_refused_during_stream_capture(ddt):
    """ddt_flush while the queue's stream is being captured returns
    DDT_ERR_STATE and leaves the requests pending (graphs capture persistent
    plans); after the capture the same requests flush normally, bit-exact,
    and later launches in the process are unaffected."""
    import torch
    spec = config1_spec()
    o = oracle.Type(spec)
    t = ddt.Type.from_spec(spec)
    src_h = random_bytes(8192, 77)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        q = ddt.Queue()
        src = torch.from_numpy(src_h).cuda()
        out = torch.full((o.size,), 0xA5, dtype=torch.uint8, device="cuda")
        q.pack(t, src, 1, out)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            with pytest.raises(ddt.DDTError) as ei:
                q.flush()
        assert ei.value.code == -2  # DDT_ERR_STATE
        assert q.flush() == 1       # still pending: flushes after the capture
        q.wait()
    assert np.array_equal(out.cpu().numpy(), oracle.pack(o, src_h))
    q.destroy()
    q2 = ddt.Queue()                # a later launch reports no stale error
    out2 = torch.full((o.size,), 0xA5, dtype=torch.uint8, device="cuda")
    q2.pack(t, src, 1, out2)
    assert q2.flush() == 1
    q2.wait()
    assert np.array_equal(out2.cpu().numpy(), oracle.pack(o, src_h))
    q2.destroy()
