"""Halo exchange plans (Alg 3, §IV-B) and the
communicator plumbing under them.  Marshalling only (csrc/halo.cpp,
csrc/comm.cpp); torch.distributed is used solely to broadcast the NCCL unique
id, to all-gather CUDA-IPC window handles and, as a host all-gather callback,
to carry the one-time plan metadata."""
from __future__ import annotations

import ctypes

from ._abi import (lib, check, P, ddt_send_t, ddt_recv_t, ddt_comm_t, ALLGATHER_FN, DDT_XCHG_NCCL,
                   DDT_XCHG_P2P, DDT_XCHG_P2P_DIRECT, DDT_XCHG_NCCL_EARLY)
from .queue import ptr_of


def torch_allgather(group=None):
    """A host all-gather over a torch.distributed group (gloo or NCCL): the
    plan-metadata path of ddt_comm_t (plumbing, never the data path)."""
    import torch.distributed as dist

    def gather(send: bytes) -> list:
        out = [None] * dist.get_world_size(group)
        dist.all_gather_object(out, send, group=group)
        return out
    return gather


def _c_allgather(gather):
    def cb(ctx, send, nbytes, recv):
        try:
            parts = gather(ctypes.string_at(send, nbytes))
            for i, b in enumerate(parts):
                assert len(b) == nbytes
                ctypes.memmove(recv + i * nbytes, b, nbytes)
            return 0
        except Exception:
            return -1
    return ALLGATHER_FN(cb)


class Windows:
    """One plan's symmetric receive windows: this rank's window (ddt_window_alloc)
    and every peer's, opened through CUDA IPC (collective over comm.gather).
    Each P2P / P2P_DIRECT plan owns its own set: flags hold the plan's epoch, so
    two plans sharing a window would read each other's signals."""

    def __init__(self, comm, nbytes: int):
        self.comm, self.nbytes = comm, int(nbytes)
        ptr = P()
        handle = ctypes.create_string_buffer(64)
        check(lib().ddt_window_alloc(comm.device, self.nbytes, ctypes.byref(ptr), handle), "ddt_window_alloc")
        self.own = ptr.value
        self._opened = []
        ptrs = [0] * comm.nranks
        ptrs[comm.rank] = ptr.value
        if comm.nranks > 1:
            import pickle
            allh = [pickle.loads(b) for b in comm.gather(pickle.dumps((bytes(handle.raw), self.nbytes)))]
            for p, (h, nb) in enumerate(allh):
                if p == comm.rank:
                    continue
                q = P()
                check(lib().ddt_window_open(comm.device, ctypes.create_string_buffer(h, 64), ctypes.byref(q)),
                      "ddt_window_open")
                ptrs[p] = q.value
                self._opened.append(q.value)
        self.peer_ptrs = (P * comm.nranks)(*ptrs)

    def close(self):
        """Every rank must have finished its last exchange on the plan first."""
        for q in self._opened:
            lib().ddt_window_close(ctypes.c_void_p(q))
        self._opened = []
        if self.own:
            lib().ddt_window_free(ctypes.c_void_p(self.own))
            self.own = None


class Comm:
    """rank / nranks, the host all-gather used for plan metadata and window
    handles, and an NCCL communicator (nranks > 1, NCCL mode)."""

    def __init__(self, rank: int = 0, nranks: int = 1, device: int = 0, nccl_comm=None, group=None, gather=None):
        self.rank, self.nranks, self.device = int(rank), int(nranks), int(device)
        self.nccl_comm = nccl_comm
        self.group = group
        self.gather = gather        # python all-gather of bytes (metadata plumbing)
        self._cb = _c_allgather(gather) if gather is not None else None

    @staticmethod
    def single(device: int = 0, nccl: bool = False) -> "Comm":
        """One rank.  nccl=True also creates a 1-rank NCCL communicator (NCCL
        send/recv to self: the DDT_SELF_VIA_NCCL test hook routes self messages
        through the NCCL-mode staging + transfer path on one GPU)."""
        c = Comm(0, 1, device)
        if nccl:
            uid = ctypes.create_string_buffer(128)
            check(lib().ddt_nccl_unique_id(uid), "ddt_nccl_unique_id")
            comm = P()
            import torch
            with torch.cuda.device(device):
                check(lib().ddt_nccl_comm_create(1, uid, 0, ctypes.byref(comm)), "ddt_nccl_comm_create")
            c.nccl_comm = comm
        return c

    @staticmethod
    def from_torch(device: int, group=None, nccl: bool = True) -> "Comm":
        """One process per GPU under torch.distributed: plan metadata travels by
        host all-gather over the group; with nccl=True an NCCL communicator of
        the same ranks is created too (unique id broadcast by the group) for the
        NCCL-mode data path."""
        import torch.distributed as dist
        rank, n = dist.get_rank(group), dist.get_world_size(group)
        c = Comm(rank, n, device, group=group, gather=torch_allgather(group) if n > 1 else None)
        if n > 1 and nccl:
            uid = ctypes.create_string_buffer(128)
            if rank == 0:
                check(lib().ddt_nccl_unique_id(uid), "ddt_nccl_unique_id")
            obj = [bytes(uid.raw) if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0, group=group)
            uid = ctypes.create_string_buffer(obj[0], 128)
            comm = P()
            import torch
            with torch.cuda.device(device):
                check(lib().ddt_nccl_comm_create(n, uid, rank, ctypes.byref(comm)), "ddt_nccl_comm_create")
            c.nccl_comm = comm
        return c

    def as_struct(self, windows=None) -> ddt_comm_t:
        c = ddt_comm_t()
        c.rank, c.nranks = self.rank, self.nranks
        c.nccl_comm = self.nccl_comm.value if isinstance(self.nccl_comm, P) else self.nccl_comm
        if windows is not None:
            c.peer_windows = ctypes.cast(windows.peer_ptrs, ctypes.POINTER(P))
            c.window_bytes = windows.nbytes
        if self._cb is not None:
            c.host_allgather = self._cb
        return c

    def close(self):
        if self.nccl_comm is not None:
            lib().ddt_nccl_comm_destroy(self.nccl_comm)
            self.nccl_comm = None


def _msgs(items, cls):
    arr = (cls * max(1, len(items)))()
    for i, m in enumerate(items):
        peer, tag, t, buf, count = m
        arr[i].peer, arr[i].tag, arr[i].type = int(peer), int(tag), t.handle.value
        arr[i].buf, arr[i].count = ptr_of(buf), int(count)
    return arr


class Halo:
    """A persistent exchange plan.  sends / recvs: lists of
    (peer, tag, Type, buffer, count); a send to (peer, tag) matches the peer's
    receive from (this rank, tag).  mode: "nccl" (fused pack -> NCCL send/recv
    -> fused unpack), "nccl_early" (the same, each peer's send/recv started as
    soon as that peer's messages are packed), "p2p" (one kernel through peers'
    windows) or "p2p_direct" (one pack-free kernel writing peers' receive
    buffers)."""

    def __init__(self, queue, comm: Comm, sends, recvs, mode: str = "nccl", graph: bool = True):
        self.queue, self.comm = queue, comm
        self._keep = [m[2] for m in sends] + [m[2] for m in recvs]
        s_arr = _msgs(sends, ddt_send_t)
        r_arr = _msgs(recvs, ddt_recv_t)
        self.mode = {"nccl": DDT_XCHG_NCCL, "p2p": DDT_XCHG_P2P, "p2p_direct": DDT_XCHG_P2P_DIRECT,
                     "nccl_early": DDT_XCHG_NCCL_EARLY}[mode]
        self.windows = None
        if self.mode in (DDT_XCHG_P2P, DDT_XCHG_P2P_DIRECT):
            nb = ctypes.c_int64()
            check(lib().ddt_halo_window_bytes(len(recvs), r_arr, ctypes.byref(nb)), "ddt_halo_window_bytes")
            self.windows = Windows(comm, nb.value)
        cs = comm.as_struct(self.windows)
        out = P()
        try:
            check(lib().ddt_halo_create(queue.handle, ctypes.byref(cs), len(sends), s_arr, len(recvs), r_arr,
                                        self.mode, ctypes.byref(out)), "ddt_halo_create")
        except Exception:
            if self.windows is not None:
                self.windows.close()
                self.windows = None
            raise
        self._h = out
        check(lib().ddt_halo_set_graph(self._h, 1 if graph else 0), "ddt_halo_set_graph")

    def exchange(self):
        check(lib().ddt_exchange(self._h), "ddt_exchange")

    def trace(self, capacity: int = 4096):
        """Start tracing the fused exchange kernel into a device buffer; returns a
        reader: reader() -> structured numpy array of per-item records."""
        import numpy as np
        import torch
        buf = torch.zeros(capacity * 48, dtype=torch.uint8, device=f"cuda:{self.queue.device}")
        check(lib().ddt_halo_set_trace(self._h, ctypes.c_void_p(buf.data_ptr()), int(capacity)), "ddt_halo_set_trace")
        self._trace_buf = buf
        dt = np.dtype([("cta", "<u4"), ("item", "<u4"), ("req", "<u4"), ("op", "<u4"),
                       ("t0", "<u8"), ("t1", "<u8"), ("t2", "<u8"), ("t3", "<u8")])

        def read():
            torch.cuda.synchronize()
            rec = buf.cpu().numpy().view(dt)
            return rec[rec["t3"] > 0]
        return read

    def set_timeout(self, seconds: float):
        """Bound of the device-side flag waits (DDT_ERR_TIMEOUT instead of a hang)."""
        check(lib().ddt_halo_set_timeout(self._h, int(seconds * 1e9)), "ddt_halo_set_timeout")

    @property
    def launches_per_exchange(self) -> int:
        v = ctypes.c_int32()
        check(lib().ddt_halo_launches_per_exchange(self._h, ctypes.byref(v)), "ddt_halo_launches_per_exchange")
        return v.value

    def destroy(self):
        """Frees the plan and its windows: every rank must have finished its last
        exchange on this plan (synchronize + barrier) before any rank destroys it."""
        if self._h and self._h.value:
            check(lib().ddt_halo_destroy(self._h), "ddt_halo_destroy")
        self._h = P()
        if getattr(self, "windows", None) is not None:
            self.windows.close()
            self.windows = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass
