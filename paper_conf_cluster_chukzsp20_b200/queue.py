"""Request list + scheduler (§IV-A): enqueue -> uid, flush
-> one fused launch, query by uid, wait.  Marshalling only (csrc/queue.cpp)."""
from __future__ import annotations

import ctypes

from ._abi import lib, check, P, ddt_queue_stats_t, STATE_NAMES


def ptr_of(buf) -> int:
    """Device address of a buffer: an int, a torch tensor, or (buffer, byte_offset)."""
    if isinstance(buf, tuple):
        base, off = buf
        return ptr_of(base) + int(off)
    if isinstance(buf, int):
        return buf
    if hasattr(buf, "data_ptr"):
        return int(buf.data_ptr())
    raise TypeError(f"cannot take a device pointer of {type(buf)!r}")


def current_stream_handle(device=None) -> int:
    import torch
    return int(torch.cuda.current_stream(device).cuda_stream)


class Queue:
    """A request list bound to (device, CUDA stream).  Default stream: torch's
    current stream on `device` at construction time."""

    def __init__(self, device: int | None = None, stream=None, capacity: int = 0):
        import torch
        if device is None:
            device = torch.cuda.current_device()
        if stream is None:
            stream = torch.cuda.current_stream(device)
        self.device = int(device)
        self.stream = stream
        handle = int(stream.cuda_stream) if hasattr(stream, "cuda_stream") else int(stream)
        out = P()
        self._lib = lib()
        check(self._lib.ddt_queue_create(self.device, ctypes.c_void_p(handle), int(capacity), ctypes.byref(out)),
              "ddt_queue_create")
        self._h = out

    @property
    def handle(self):
        return self._h

    def pack(self, t, src, count: int, dst_packed) -> int:
        """Scheduler (1): enqueue a packing request; returns its uid."""
        rc = self._lib.ddt_pack_enqueue(self._h, t.handle, ptr_of(src), count, ptr_of(dst_packed))
        return rc if rc >= 0 else check(rc, "ddt_pack_enqueue")

    def unpack(self, t, src_packed, count: int, dst) -> int:
        """Scheduler (1): enqueue an unpacking request; returns its uid."""
        rc = self._lib.ddt_unpack_enqueue(self._h, t.handle, ptr_of(src_packed), count, ptr_of(dst))
        return rc if rc >= 0 else check(rc, "ddt_unpack_enqueue")

    def direct(self, src_type, src, src_count: int, dst_type, dst, dst_count: int) -> int:
        """Enqueue a DirectIPC request: gather through src_type, scatter through
        dst_type, no packed intermediate."""
        return check(lib().ddt_direct_enqueue(self._h, src_type.handle, ctypes.c_void_p(ptr_of(src)), int(src_count),
                                              dst_type.handle, ctypes.c_void_p(ptr_of(dst)), int(dst_count)),
                     "ddt_direct_enqueue")

    def enqueue_many(self, op: str, types, srcs, counts, dsts):
        """Bulk enqueue (ddt_enqueue_many): op 'pack' | 'unpack'; types a Type or
        a sequence of n Types; srcs / dsts sequences of n buffers; counts an int
        or n ints.  Returns the uids (numpy int64).  Raises on the first failed
        request (requests before it stay enqueued); try_enqueue_many reports it."""
        k, uids = self.try_enqueue_many(op, types, srcs, counts, dsts)
        if k < len(uids):
            check(int(uids[k]), f"ddt_enqueue_many (request {k})")
        return uids

    def try_enqueue_many(self, op: str, types, srcs, counts, dsts):
        """Like enqueue_many but returns (k, uids): k requests were enqueued; if
        k < n, uids[k] is request k's negative status (e.g. -3 = queue full:
        flush and resubmit from k)."""
        import numpy as np
        n = len(srcs)
        tys = np.asarray([t.handle.value for t in types] if isinstance(types, (list, tuple))
                         else [types.handle.value] * n, dtype=np.uint64)
        s = np.asarray([ptr_of(b) for b in srcs], dtype=np.uint64)
        d = np.asarray([ptr_of(b) for b in dsts], dtype=np.uint64)
        c = np.asarray(counts if isinstance(counts, (list, tuple, np.ndarray)) else [counts] * n, dtype=np.int64)
        return self.enqueue_many_raw(0 if op == "pack" else 1, tys, s, c, d)

    def enqueue_many_raw(self, op: int, tys, srcs, counts, dsts):
        """ddt_enqueue_many over prepared numpy arrays (uint64 handles / pointers,
        int64 counts): one call across the ABI for the whole batch.  Returns
        (k, uids) as try_enqueue_many."""
        import numpy as np
        n = len(srcs)
        uids = np.empty(n, dtype=np.int64)
        k = self._lib.ddt_enqueue_many(self._h, int(op), n, tys.ctypes.data, srcs.ctypes.data, counts.ctypes.data,
                                       dsts.ctypes.data, uids.ctypes.data)
        if k < 0:
            check(k, "ddt_enqueue_many")
        return int(k), uids

    def try_pack(self, t, src, count, dst_packed) -> int:
        """Like pack() but returns the negative status instead of raising."""
        return lib().ddt_pack_enqueue(self._h, t.handle, ctypes.c_void_p(ptr_of(src)), int(count),
                                      ctypes.c_void_p(ptr_of(dst_packed)))

    def flush(self) -> int:
        """Scheduler (2): one fused launch for every pending request."""
        rc = self._lib.ddt_flush(self._h)
        return rc if rc >= 0 else check(rc, "ddt_flush")

    def query(self, uid: int) -> str:
        """Scheduler (4): 'pending' | 'busy' | 'completed'."""
        st = ctypes.c_int32()
        check(lib().ddt_query(self._h, int(uid), ctypes.byref(st)), "ddt_query")
        return STATE_NAMES[st.value]

    def wait(self):
        check(lib().ddt_wait(self._h), "ddt_wait")

    def set_flush_threshold(self, nbytes: int):
        """Auto-flush once pending requests hold >= nbytes (§IV-C); 0 = off."""
        check(self._lib.ddt_queue_set_flush_threshold(self._h, int(nbytes)), "ddt_queue_set_flush_threshold")

    def set_response_flags(self, enable: bool = True):
        """GPU-written per-request completion."""
        check(self._lib.ddt_queue_set_response_flags(self._h, 1 if enable else 0), "ddt_queue_set_response_flags")

    def stats(self) -> dict:
        s = ddt_queue_stats_t()
        check(lib().ddt_queue_get_stats(self._h, ctypes.byref(s)), "ddt_queue_get_stats")
        return {"requests": s.requests, "launches": s.launches, "flushes": s.flushes, "bytes": s.bytes,
                "phased": s.phased}

    def destroy(self):
        if self._h and self._h.value:
            check(lib().ddt_queue_destroy(self._h), "ddt_queue_destroy")
        self._h = P()

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


class Plan:
    """A persistent fused batch: the queue's pending requests frozen into a
    device work table uploaded once; launch() = one fused kernel (static-batch
    replay, the 'fused + graph replay' arm of configs[4])."""

    def __init__(self, queue: Queue):
        self.queue = queue
        out = P()
        check(lib().ddt_plan_create(queue.handle, ctypes.byref(out)), "ddt_plan_create")
        self._h = out

    def launch(self):
        check(lib().ddt_plan_launch(self._h), "ddt_plan_launch")

    def destroy(self):
        if self._h and self._h.value:
            check(lib().ddt_plan_destroy(self._h), "ddt_plan_destroy")
        self._h = P()

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass
