"""Datatype objects: MPI-3.1 §4.1 constructors and commit (Alg 1/3
lines 1-2).  Marshalling only; all logic is in libddt (csrc/types.cpp)."""
from __future__ import annotations

import ctypes

import numpy as np

from ._abi import lib, check, BASE_CODES, LAYOUT_KINDS, P


def _i64arr(v):
    a = np.ascontiguousarray(np.asarray(v, dtype=np.int64).reshape(-1))
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


class Type:
    """A library-owned datatype handle.  Children are kept alive by the library
    (reference counted), so intermediate Python objects may be dropped."""

    def __init__(self, handle, predefined=False):
        self._h = ctypes.c_void_p(handle)
        self._predefined = predefined

    # ---------------------------------------------------------- builders
    @staticmethod
    def basic(name: str) -> "Type":
        out = P()
        check(lib().ddt_type_basic(BASE_CODES[name], ctypes.byref(out)), "ddt_type_basic")
        return Type(out.value, predefined=True)

    @staticmethod
    def contiguous(count: int, old: "Type") -> "Type":
        out = P()
        check(lib().ddt_create_contiguous(int(count), old._h, ctypes.byref(out)), "ddt_create_contiguous")
        return Type(out.value)

    @staticmethod
    def vector(count: int, blocklen: int, stride: int, old: "Type") -> "Type":
        out = P()
        check(lib().ddt_create_vector(int(count), int(blocklen), int(stride), old._h, ctypes.byref(out)),
              "ddt_create_vector")
        return Type(out.value)

    @staticmethod
    def hvector(count: int, blocklen: int, stride_bytes: int, old: "Type") -> "Type":
        out = P()
        check(lib().ddt_create_hvector(int(count), int(blocklen), int(stride_bytes), old._h, ctypes.byref(out)),
              "ddt_create_hvector")
        return Type(out.value)

    @staticmethod
    def indexed(blocklens, displs, old: "Type", hindexed: bool = False) -> "Type":
        b, bp = _i64arr(blocklens)
        d, dp = _i64arr(displs)
        assert b.size == d.size
        out = P()
        f = lib().ddt_create_hindexed if hindexed else lib().ddt_create_indexed
        check(f(int(b.size), bp, dp, old._h, ctypes.byref(out)), "ddt_create_(h)indexed")
        return Type(out.value)

    @staticmethod
    def hindexed(blocklens, displs_bytes, old: "Type") -> "Type":
        return Type.indexed(blocklens, displs_bytes, old, hindexed=True)

    @staticmethod
    def indexed_block(blocklen: int, displs, old: "Type", hindexed: bool = False) -> "Type":
        d, dp = _i64arr(displs)
        out = P()
        f = lib().ddt_create_hindexed_block if hindexed else lib().ddt_create_indexed_block
        check(f(int(d.size), int(blocklen), dp, old._h, ctypes.byref(out)), "ddt_create_(h)indexed_block")
        return Type(out.value)

    @staticmethod
    def struct(blocklens, displs_bytes, types) -> "Type":
        b, bp = _i64arr(blocklens)
        d, dp = _i64arr(displs_bytes)
        assert b.size == d.size == len(types)
        arr = (ctypes.c_void_p * max(1, len(types)))(*[t._h.value for t in types])
        out = P()
        check(lib().ddt_create_struct(int(b.size), bp, dp, arr, ctypes.byref(out)), "ddt_create_struct")
        return Type(out.value)

    @staticmethod
    def resized(old: "Type", lb: int, extent: int) -> "Type":
        out = P()
        check(lib().ddt_create_resized(old._h, int(lb), int(extent), ctypes.byref(out)), "ddt_create_resized")
        return Type(out.value)

    @staticmethod
    def subarray(sizes, subsizes, starts, order: str, old: "Type") -> "Type":
        s, sp = _i64arr(sizes)
        ss, ssp = _i64arr(subsizes)
        st, stp = _i64arr(starts)
        out = P()
        check(lib().ddt_create_subarray(int(s.size), sp, ssp, stp, 0 if order == "C" else 1, old._h,
                                        ctypes.byref(out)), "ddt_create_subarray")
        return Type(out.value)

    @staticmethod
    def from_spec(spec, commit: bool = True) -> "Type":
        """Build from the neutral spec-tuple language (see ddt_inputs)."""
        t = Type._build(spec)
        if commit:
            t.commit()
        return t

    @staticmethod
    def _build(spec) -> "Type":
        if isinstance(spec, Type):
            return spec
        k = spec[0]
        if k == "basic":
            return Type.basic(spec[1])
        if k == "contiguous":
            return Type.contiguous(spec[1], Type._build(spec[2]))
        if k == "vector":
            return Type.vector(spec[1], spec[2], spec[3], Type._build(spec[4]))
        if k == "hvector":
            return Type.hvector(spec[1], spec[2], spec[3], Type._build(spec[4]))
        if k == "indexed":
            return Type.indexed(spec[1], spec[2], Type._build(spec[3]))
        if k == "hindexed":
            return Type.hindexed(spec[1], spec[2], Type._build(spec[3]))
        if k == "subarray":
            return Type.subarray(spec[1], spec[2], spec[3], spec[4], Type._build(spec[5]))
        if k == "struct":
            return Type.struct(spec[1], spec[2], [Type._build(o) for o in spec[3]])
        if k == "resized":
            return Type.resized(Type._build(spec[1]), spec[2], spec[3])
        raise ValueError(f"unknown spec kind {k!r}")

    # ---------------------------------------------------------- lifecycle
    def commit(self) -> "Type":
        check(lib().ddt_commit(self._h), "ddt_commit")
        return self

    def free(self):
        if self._h and self._h.value and not self._predefined:
            h = ctypes.c_void_p(self._h.value)
            lib().ddt_free(ctypes.byref(h))
        self._h = ctypes.c_void_p(None)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    @property
    def handle(self):
        return self._h

    # ---------------------------------------------------------- queries
    @property
    def size(self) -> int:
        v = ctypes.c_int64()
        check(lib().ddt_get_size(self._h, ctypes.byref(v)), "ddt_get_size")
        return v.value

    def extent(self):
        lb, ex = ctypes.c_int64(), ctypes.c_int64()
        check(lib().ddt_get_extent(self._h, ctypes.byref(lb), ctypes.byref(ex)), "ddt_get_extent")
        return lb.value, ex.value

    def true_extent(self):
        lb, ex = ctypes.c_int64(), ctypes.c_int64()
        check(lib().ddt_get_true_extent(self._h, ctypes.byref(lb), ctypes.byref(ex)), "ddt_get_true_extent")
        return lb.value, ex.value

    @property
    def num_segments(self) -> int:
        v = ctypes.c_int64()
        check(lib().ddt_get_num_segments(self._h, ctypes.byref(v)), "ddt_get_num_segments")
        return v.value

    @property
    def layout_kind(self) -> str:
        v = ctypes.c_int32()
        check(lib().ddt_get_layout_kind(self._h, ctypes.byref(v)), "ddt_get_layout_kind")
        return LAYOUT_KINDS[v.value]

    @property
    def overlaps(self) -> bool:
        v = ctypes.c_int32()
        check(lib().ddt_get_overlaps(self._h, ctypes.byref(v)), "ddt_get_overlaps")
        return bool(v.value)

    def segments(self):
        """(offsets, lengths) of one instance's segments in packed order."""
        n = ctypes.c_int64()
        check(lib().ddt_get_segments(self._h, None, None, 0, ctypes.byref(n)), "ddt_get_segments")
        o = np.zeros(max(n.value, 1), np.int64)
        ln = np.zeros(max(n.value, 1), np.int64)
        check(lib().ddt_get_segments(self._h, o.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                     ln.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), n.value, ctypes.byref(n)),
              "ddt_get_segments")
        return o[:n.value], ln[:n.value]
