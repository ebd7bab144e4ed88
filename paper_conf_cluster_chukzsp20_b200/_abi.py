"""ctypes prototypes of include/ddt.h (argument marshalling only)."""
from __future__ import annotations

import ctypes
import os
import threading

HERE = os.path.dirname(os.path.abspath(__file__))
# DDT_LIBDDT: load another build of the library (A/B experiments only)
LIB_PATH = os.environ.get("DDT_LIBDDT") or os.path.join(HERE, "libddt.so")

DDT_OK = 0
ERRORS = {
    -1: "DDT_ERR_ARG", -2: "DDT_ERR_STATE", -3: "DDT_ERR_QUEUE_FULL", -4: "DDT_ERR_OVERLAP",
    -5: "DDT_ERR_NOMEM", -6: "DDT_ERR_CUDA", -7: "DDT_ERR_NCCL", -8: "DDT_ERR_SIZE_MISMATCH",
    -9: "DDT_ERR_TIMEOUT", -10: "DDT_ERR_UNSUPPORTED", -11: "DDT_ERR_NODEV",
}
BASE_CODES = {"byte": 0, "int32": 1, "int64": 2, "float": 3, "double": 4}
LAYOUT_KINDS = {0: "empty", 1: "strided", 2: "uniform_list", 3: "general_list"}
STATE_NAMES = {0: "idle", 1: "pending", 2: "busy", 3: "completed"}
DDT_PENDING, DDT_BUSY, DDT_COMPLETED = 1, 2, 3
DDT_XCHG_NCCL, DDT_XCHG_P2P, DDT_XCHG_P2P_DIRECT, DDT_XCHG_NCCL_EARLY = 0, 1, 2, 3

c_type_p = ctypes.c_void_p
I64, I32, P = ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p
I64P = ctypes.POINTER(ctypes.c_int64)
I32P = ctypes.POINTER(ctypes.c_int32)


class ddt_send_t(ctypes.Structure):
    _fields_ = [("peer", I32), ("tag", I32), ("type", P), ("buf", P), ("count", I64)]


class ddt_recv_t(ctypes.Structure):
    _fields_ = [("peer", I32), ("tag", I32), ("type", P), ("buf", P), ("count", I64)]


ALLGATHER_FN = ctypes.CFUNCTYPE(I32, P, P, I64, P)


class ddt_comm_t(ctypes.Structure):
    _fields_ = [("rank", I32), ("nranks", I32), ("nccl_comm", P), ("peer_windows", ctypes.POINTER(P)),
                ("window_bytes", I64), ("host_allgather", ALLGATHER_FN), ("host_ctx", P)]


class ddt_queue_stats_t(ctypes.Structure):
    _fields_ = [("requests", I64), ("launches", I64), ("flushes", I64), ("bytes", I64), ("phased", I64)]


# name -> (restype, argtypes); the complete list of exported entry points
PROTOTYPES = {
    "ddt_type_basic": (I32, [ctypes.c_int, ctypes.POINTER(P)]),
    "ddt_create_contiguous": (I32, [I64, P, ctypes.POINTER(P)]),
    "ddt_create_vector": (I32, [I64, I64, I64, P, ctypes.POINTER(P)]),
    "ddt_create_hvector": (I32, [I64, I64, I64, P, ctypes.POINTER(P)]),
    "ddt_create_indexed": (I32, [I64, I64P, I64P, P, ctypes.POINTER(P)]),
    "ddt_create_hindexed": (I32, [I64, I64P, I64P, P, ctypes.POINTER(P)]),
    "ddt_create_indexed_block": (I32, [I64, I64, I64P, P, ctypes.POINTER(P)]),
    "ddt_create_hindexed_block": (I32, [I64, I64, I64P, P, ctypes.POINTER(P)]),
    "ddt_create_struct": (I32, [I64, I64P, I64P, ctypes.POINTER(P), ctypes.POINTER(P)]),
    "ddt_create_resized": (I32, [P, I64, I64, ctypes.POINTER(P)]),
    "ddt_create_subarray": (I32, [ctypes.c_int, I64P, I64P, I64P, ctypes.c_int, P, ctypes.POINTER(P)]),
    "ddt_commit": (I32, [P]),
    "ddt_free": (I32, [ctypes.POINTER(P)]),
    "ddt_get_size": (I32, [P, I64P]),
    "ddt_get_extent": (I32, [P, I64P, I64P]),
    "ddt_get_true_extent": (I32, [P, I64P, I64P]),
    "ddt_get_num_segments": (I32, [P, I64P]),
    "ddt_get_layout_kind": (I32, [P, I32P]),
    "ddt_get_segments": (I32, [P, I64P, I64P, I64, I64P]),
    "ddt_get_overlaps": (I32, [P, I32P]),
    "ddt_queue_create": (I32, [ctypes.c_int, P, I32, ctypes.POINTER(P)]),
    "ddt_queue_destroy": (I32, [P]),
    "ddt_pack_enqueue": (I64, [P, P, P, I64, P]),
    "ddt_unpack_enqueue": (I64, [P, P, P, I64, P]),
    "ddt_direct_enqueue": (I64, [P, P, P, I64, P, P, I64]),
    "ddt_enqueue_many": (I64, [P, I32, I64, P, P, P, P, P]),
    "ddt_flush": (I32, [P]),
    "ddt_query": (I32, [P, I64, I32P]),
    "ddt_wait": (I32, [P]),
    "ddt_queue_get_stats": (I32, [P, ctypes.POINTER(ddt_queue_stats_t)]),
    "ddt_queue_set_flush_threshold": (I32, [P, I64]),
    "ddt_queue_set_response_flags": (I32, [P, I32]),
    "ddt_plan_create": (I32, [P, ctypes.POINTER(P)]),
    "ddt_plan_launch": (I32, [P]),
    "ddt_plan_destroy": (I32, [P]),
    "ddt_halo_window_bytes": (I32, [I32, ctypes.POINTER(ddt_recv_t), I64P]),
    "ddt_halo_create": (I32, [P, ctypes.POINTER(ddt_comm_t), I32, ctypes.POINTER(ddt_send_t), I32,
                              ctypes.POINTER(ddt_recv_t), I32, ctypes.POINTER(P)]),
    "ddt_exchange": (I32, [P]),
    "ddt_halo_set_graph": (I32, [P, I32]),
    "ddt_halo_set_timeout": (I32, [P, I64]),
    "ddt_halo_set_trace": (I32, [P, P, I64]),
    "ddt_halo_launches_per_exchange": (I32, [P, I32P]),
    "ddt_halo_destroy": (I32, [P]),
    "ddt_nccl_unique_id": (I32, [P]),
    "ddt_nccl_comm_create": (I32, [I32, P, I32, ctypes.POINTER(P)]),
    "ddt_nccl_comm_destroy": (I32, [P]),
    "ddt_window_alloc": (I32, [ctypes.c_int, I64, ctypes.POINTER(P), P]),
    "ddt_window_open": (I32, [ctypes.c_int, P, ctypes.POINTER(P)]),
    "ddt_window_close": (I32, [P]),
    "ddt_window_free": (I32, [P]),
    "ddt_strerror": (ctypes.c_char_p, [I32]),
    "ddt_last_error_message": (ctypes.c_char_p, []),
    "ddt_version": (I32, []),
    "ddt_reload_env": (None, []),
    "ddt_built_sm": (I32, []),
}

_lock = threading.Lock()
_lib = None


class DDTError(RuntimeError):
    def __init__(self, code: int, where: str = ""):
        self.code = int(code)
        name = ERRORS.get(self.code, str(code))
        detail = ""
        try:
            L = lib()
            detail = (L.ddt_last_error_message() or b"").decode(errors="replace")
            msg = (L.ddt_strerror(self.code) or b"").decode()
        except Exception:
            msg = ""
        super().__init__(f"{where}: {name} ({msg}){' -- ' + detail if detail else ''}")


def lib():
    """Load libddt.so (raises if it has not been built: no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(f"{LIB_PATH} not built; run `python -m paper_conf_cluster_chukzsp20_b200.build`")
            L = ctypes.CDLL(LIB_PATH)
            for name, (res, args) in PROTOTYPES.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def check(rc: int, where: str) -> int:
    if rc < 0:
        raise DDTError(rc, where)
    return rc
