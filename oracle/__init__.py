"""CPU oracle for MPI derived-datatype pack / unpack -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  The product package
(``paper_conf_cluster_chukzsp20_b200``) never imports it, and it never imports the
product: the two share no code.  The only shared module is ``ddt_inputs`` (seeded
input generators and workload recipes, no datatype arithmetic).

The arithmetic lives in ``ddt_oracle.c`` (plain C99, nested loops over the MPI
typemap, see its header for the PAPER.md / MPI-3.1 passages it follows).  This
module only marshals arguments into it:

* ``Type(spec)``           -- build the constructor tree from a spec tuple
* ``size / extent / true_extent / typemap`` -- enumerated queries
* ``pack / unpack``        -- MPI_Pack / MPI_Unpack semantics (Alg 1,
                              P:98-119; §IV-A.1)
* ``run_batch``            -- a fused batch executed sequentially in enqueue
                              order (equal to any concurrent
                              order under the non-aliasing precondition, DESIGN R6)
* ``exchange``             -- all ranks of a halo exchange simulated in one
                              process: for each message, unpack(pack(...))
                              (Alg 3)

Spec tuples (the neutral input language both sides parse independently):
    ("basic", "byte"|"int32"|"int64"|"float"|"double")
    ("contiguous", n, old)
    ("vector", count, blocklen, stride, old)
    ("hvector", count, blocklen, stride_bytes, old)
    ("indexed", blocklens, displs, old)
    ("hindexed", blocklens, displs_bytes, old)
    ("subarray", sizes, subsizes, starts, "C"|"F", old)
    ("struct", blocklens, displs_bytes, [old_0, old_1, ...])
    ("resized", old, lb, extent)

Parity status: every function here is pinned by tests/test_oracle_pins.py
(numpy slicing / as_strided / concatenation, closed forms incl. oldtypes with
lb != 0, numpy align=True records for the struct alignment epsilon,
brute-force self-describing buffers, round-trip invariants, the config-1 and
struct-alignment golden files; run_batch by numpy slicing / assignment on
shared buffers).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ddt_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

BASIC_SIZES = {"byte": 1, "int32": 4, "int64": 8, "float": 4, "double": 8}

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with plain gcc (-O2, no vectorisation tricks)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-std=c99", "-O2", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            P, I64, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
            I64P = ctypes.POINTER(ctypes.c_int64)
            for name, args in {
                "orc_basic": [I64],
                "orc_contiguous": [I64, P],
                "orc_vector": [I64, I64, I64, P],
                "orc_hvector": [I64, I64, I64, P],
                "orc_indexed": [I64, I64P, I64P, P],
                "orc_hindexed": [I64, I64P, I64P, P],
                "orc_subarray": [I, I64P, I64P, I64P, I, P],
                "orc_struct": [I64, I64P, I64P, ctypes.POINTER(P)],
                "orc_resized": [P, I64, I64],
            }.items():
                f = getattr(L, name)
                f.argtypes = args
                f.restype = P
            L.orc_free.argtypes = [P]
            L.orc_free.restype = None
            L.orc_size.argtypes = [P]
            L.orc_size.restype = I64
            L.orc_num_entries.argtypes = [P]
            L.orc_num_entries.restype = I64
            L.orc_get_extent.argtypes = [P, I64P, I64P]
            L.orc_get_extent.restype = None
            L.orc_get_true_extent.argtypes = [P, I64P, I64P]
            L.orc_get_true_extent.restype = None
            L.orc_typemap.argtypes = [P, I64, I64P, I64P, I64]
            L.orc_typemap.restype = I64
            L.orc_pack.argtypes = [P, P, I64, P]
            L.orc_pack.restype = I64
            L.orc_unpack.argtypes = [P, P, I64, P]
            L.orc_unpack.restype = I64
            _lib = L
    return _lib


def _arr(v):
    a = (ctypes.c_int64 * max(1, len(v)))(*[int(x) for x in v])
    return a


class Type:
    """An oracle datatype built from a spec tuple (keeps its subtree alive)."""

    def __init__(self, spec):
        self.spec = spec
        L = lib()
        kind = spec[0]
        self.children = []
        self._keep = []
        if kind == "basic":
            self.ptr = L.orc_basic(BASIC_SIZES[spec[1]])
        elif kind == "contiguous":
            old = self._child(spec[2])
            self.ptr = L.orc_contiguous(int(spec[1]), old.ptr)
        elif kind == "vector":
            old = self._child(spec[4])
            self.ptr = L.orc_vector(int(spec[1]), int(spec[2]), int(spec[3]), old.ptr)
        elif kind == "hvector":
            old = self._child(spec[4])
            self.ptr = L.orc_hvector(int(spec[1]), int(spec[2]), int(spec[3]), old.ptr)
        elif kind in ("indexed", "hindexed"):
            bl, d = list(spec[1]), list(spec[2])
            assert len(bl) == len(d)
            old = self._child(spec[3])
            a, b = _arr(bl), _arr(d)
            self._keep += [a, b]
            f = L.orc_indexed if kind == "indexed" else L.orc_hindexed
            self.ptr = f(len(bl), a, b, old.ptr)
        elif kind == "struct":
            bl, d, olds = list(spec[1]), list(spec[2]), list(spec[3])
            assert len(bl) == len(d) == len(olds)
            kids = [self._child(o) for o in olds]
            a, b = _arr(bl), _arr(d)
            tp = (ctypes.c_void_p * max(1, len(kids)))(*[k.ptr for k in kids])
            self._keep += [a, b, tp]
            self.ptr = L.orc_struct(len(bl), a, b, tp)
        elif kind == "resized":
            old = self._child(spec[1])
            self.ptr = L.orc_resized(old.ptr, int(spec[2]), int(spec[3]))
        elif kind == "subarray":
            sizes, subsizes, starts, order = spec[1], spec[2], spec[3], spec[4]
            old = self._child(spec[5])
            nd = len(sizes)
            a, b, c = _arr(sizes), _arr(subsizes), _arr(starts)
            self._keep += [a, b, c]
            self.ptr = L.orc_subarray(nd, a, b, c, 0 if order == "C" else 1, old.ptr)
        else:
            raise ValueError(f"unknown spec kind {kind!r}")
        if not self.ptr:
            raise ValueError(f"oracle rejected spec {spec!r}")

    def _child(self, spec):
        c = spec if isinstance(spec, Type) else Type(spec)
        self.children.append(c)
        return c

    def __del__(self):
        try:
            if getattr(self, "ptr", None):
                lib().orc_free(self.ptr)
        except Exception:
            pass

    # -- enumerated queries --------------------------------------------
    @property
    def size(self) -> int:
        return int(lib().orc_size(self.ptr))

    @property
    def num_entries(self) -> int:
        return int(lib().orc_num_entries(self.ptr))

    def extent(self):
        lb, ex = ctypes.c_int64(), ctypes.c_int64()
        lib().orc_get_extent(self.ptr, ctypes.byref(lb), ctypes.byref(ex))
        return lb.value, ex.value

    def true_extent(self):
        lb, ex = ctypes.c_int64(), ctypes.c_int64()
        lib().orc_get_true_extent(self.ptr, ctypes.byref(lb), ctypes.byref(ex))
        return lb.value, ex.value

    def typemap(self, count: int = 1):
        """(disp, nbytes) of every basic entry of `count` instances, typemap order."""
        n = int(lib().orc_typemap(self.ptr, count, None, None, 0))
        d = np.zeros(max(n, 1), dtype=np.int64)
        ln = np.zeros(max(n, 1), dtype=np.int64)
        lib().orc_typemap(self.ptr, count,
                          d.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                          ln.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), n)
        return d[:n], ln[:n]

    def footprint(self, count: int = 1):
        """(min_byte, max_byte_exclusive) touched by `count` instances (0,0 if empty)."""
        d, ln = self.typemap(count)
        if len(d) == 0:
            return 0, 0
        return int(d.min()), int((d + ln).max())


def _ptr(buf: np.ndarray, byte_offset: int = 0):
    assert buf.flags["C_CONTIGUOUS"]
    return ctypes.c_void_p(buf.ctypes.data + int(byte_offset))


def pack(t: Type, src: np.ndarray, count: int = 1, src_offset: int = 0) -> np.ndarray:
    """MPI_Pack of `count` instances; `src_offset` = byte position of the MPI
    buffer address inside `src` (so negative displacements stay in bounds)."""
    out = np.empty(count * t.size, dtype=np.uint8)
    src_u8 = src.view(np.uint8).reshape(-1)
    lo, hi = t.footprint(count)
    if count * t.size:
        assert src_offset + lo >= 0 and src_offset + hi <= src_u8.nbytes, "footprint out of bounds"
    n = lib().orc_pack(t.ptr, _ptr(src_u8, src_offset), count, _ptr(out))
    assert n == out.nbytes
    return out


def unpack(t: Type, packed: np.ndarray, dst: np.ndarray, count: int = 1, dst_offset: int = 0) -> None:
    """MPI_Unpack of `count` instances into `dst` (in place)."""
    pk = np.ascontiguousarray(packed).view(np.uint8).reshape(-1)
    assert pk.nbytes >= count * t.size
    dst_u8 = dst.view(np.uint8).reshape(-1)
    lo, hi = t.footprint(count)
    if count * t.size:
        assert dst_offset + lo >= 0 and dst_offset + hi <= dst_u8.nbytes, "footprint out of bounds"
    n = lib().orc_unpack(t.ptr, _ptr(pk), count, _ptr(dst_u8, dst_offset))
    assert n == count * t.size


def run_batch(requests):
    """Execute a batch sequentially in enqueue order.

    requests: list of dicts {op: "pack"|"unpack", type: Type, count, src, src_offset,
    dst, dst_offset}; src/dst are uint8 numpy arrays modified in place."""
    for r in requests:
        t, c = r["type"], r["count"]
        if r["op"] == "pack":
            out = pack(t, r["src"], c, r.get("src_offset", 0))
            d = r["dst"].view(np.uint8).reshape(-1)
            o = r.get("dst_offset", 0)
            d[o:o + out.nbytes] = out
        else:
            s = r["src"].view(np.uint8).reshape(-1)
            o = r.get("src_offset", 0)
            unpack(t, s[o:o + c * t.size], r["dst"], c, r.get("dst_offset", 0))


def exchange(arrays, messages):
    """Simulate one halo exchange of all ranks in one process.

    arrays:   {(rank, var): numpy array} -- modified in place.
    messages: list of dicts {src_rank, dst_rank, var, send: Type, recv: Type}
              (one boundary buffer per message, Alg 3).
    All packs read the pre-exchange state (the sends are posted before any
    receive completes), then every message is unpacked."""
    packed = []
    for m in messages:
        packed.append(pack(m["send"], arrays[(m["src_rank"], m["var"])]))
    for m, p in zip(messages, packed):
        unpack(m["recv"], p, arrays[(m["dst_rank"], m["var"])])
